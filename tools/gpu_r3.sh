# router + M1 directory check. bash tools/gpu_r3.sh TAG
TAG=${1:-r3}
mkdir -p gpurun_out
python tools/build.py > gpurun_out/build_$TAG.log 2>&1 || { echo build failed; exit 1; }
timeout 900 python -m pytest tests/test_shard_gpu.py -x -q -p no:cacheprovider > gpurun_out/pytest_$TAG.log 2>&1
echo "pytest rc=$?" >> gpurun_out/pytest_$TAG.log
for r in C5z:lib C5u:lib C2:lib C2:wire; do
  cfg=${r%%:*}; plane=${r##*:}; ex=""
  if [ $plane = wire ]; then plane=lib; ex="SEPO_SHARD_WIRE=1"; fi
  env $ex timeout 600 python bench.py --route --plane $plane --config $cfg --steps 5 --warmup 3 --e2e-steps 1 \
      > gpurun_out/routed_${TAG}_${r/:/_}.log 2>&1
  echo "$r rc=$?" >> gpurun_out/routed_${TAG}.txt
done
AB_SPECS="C2 0.5" bash tools/ab.sh nb_$TAG "SEPO_BENCH_NB_IB=2" "SEPO_BENCH_NB_IB=4" "SEPO_BENCH_NB_IB=8"
echo done
