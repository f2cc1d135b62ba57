# peer-memory exchange: tests + routed lines (p2p on / off). bash tools/gpu_r8.sh TAG
TAG=${1:-r8}
mkdir -p gpurun_out
python tools/build.py > gpurun_out/build_$TAG.log 2>&1 || { echo build failed; exit 1; }
timeout 900 python -m pytest tests/test_shard_gpu.py -x -q -p no:cacheprovider > gpurun_out/pytest_$TAG.log 2>&1
echo "pytest rc=$?" >> gpurun_out/pytest_$TAG.log
for r in C5z:1 C2:1 C5z:0 C2:0; do
  cfg=${r%%:*}; p=${r##*:}
  SEPO_SHARD_P2P=$p timeout 600 python bench.py --route --plane lib --config $cfg --steps 5 --warmup 3 --e2e-steps 1 \
      > gpurun_out/routed_${TAG}_${cfg}_p2p$p.log 2>&1
  echo "$r rc=$?" >> gpurun_out/routed_${TAG}.txt
done
echo done
