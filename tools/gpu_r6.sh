# router + dir-prefetch parity, routed launch list, routed lines, M1 timing. bash tools/gpu_r6.sh TAG
TAG=${1:-r6}
mkdir -p gpurun_out
python tools/build.py > gpurun_out/build_$TAG.log 2>&1 || { echo build failed; exit 1; }
timeout 900 python -m pytest tests/test_shard_gpu.py tests/test_hot_parity_gpu.py -x -q -p no:cacheprovider > gpurun_out/pytest_$TAG.log 2>&1
echo "pytest rc=$?" >> gpurun_out/pytest_$TAG.log
timeout 300 python tools/time_job.py C2 0.5 > gpurun_out/m1_$TAG.json 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/routed_launches_$TAG.csv \
   python bench.py --route --plane lib --config C5z --scale 0.125 --steps 1 --warmup 1 --e2e-steps 0 > gpurun_out/routed_ncu_$TAG.log 2>&1
for r in C5z:lib C5z:torch C2:torch C2:lib; do
  cfg=${r%%:*}; plane=${r##*:}
  timeout 600 python bench.py --route --plane $plane --config $cfg --steps 5 --warmup 3 --e2e-steps 1 \
      > gpurun_out/routed_${TAG}_${r/:/_}.log 2>&1
  echo "$r rc=$?" >> gpurun_out/routed_${TAG}.txt
done
echo done
