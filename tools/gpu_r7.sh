# sharded tests, routed lines at the default chunk, unrouted C5z / C2 for comparison. bash tools/gpu_r7.sh TAG
TAG=${1:-r7}
mkdir -p gpurun_out
python tools/build.py > gpurun_out/build_$TAG.log 2>&1 || { echo build failed; exit 1; }
timeout 900 python -m pytest tests/test_shard_gpu.py -x -q -p no:cacheprovider > gpurun_out/pytest_$TAG.log 2>&1
echo "pytest rc=$?" >> gpurun_out/pytest_$TAG.log
for r in C5z:lib C2:lib; do
  cfg=${r%%:*}; plane=${r##*:}
  timeout 600 python bench.py --route --plane $plane --config $cfg --steps 5 --warmup 3 --e2e-steps 1 \
      > gpurun_out/routed_${TAG}_${r/:/_}.log 2>&1
  echo "$r rc=$?" >> gpurun_out/routed_${TAG}.txt
done
timeout 600 python tools/time_job.py C5z 4 > gpurun_out/unrouted_${TAG}_C5z.json 2>&1
timeout 600 python tools/time_job.py C5u 4 0.125 > gpurun_out/unrouted_${TAG}_C5u8.json 2>&1
timeout 600 python tools/time_job.py C2 4 > gpurun_out/unrouted_${TAG}_C2.json 2>&1
echo done
