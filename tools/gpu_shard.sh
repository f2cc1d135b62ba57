# sharded-job check on one GPU: tests of the router / NCCL plane, routed bench lines at N = 1.
#   bash tools/gpu_shard.sh TAG "CFG:PLANE ..."
TAG=${1:-sh}
RUNS=${2:-"C2:lib C2:torch C5z:lib C5z:torch C5u:lib C5u:torch C3:lib C3:torch"}
mkdir -p gpurun_out
python tools/build.py > gpurun_out/build_$TAG.log 2>&1 || { echo build failed; exit 1; }
timeout 900 python -m pytest tests/test_shard_gpu.py -x -q -p no:cacheprovider > gpurun_out/pytest_$TAG.log 2>&1
echo "pytest rc=$?" >> gpurun_out/pytest_$TAG.log
for r in $RUNS; do
  cfg=${r%%:*}; plane=${r##*:}
  timeout 600 python bench.py --route --plane $plane --config $cfg --steps 5 --warmup 3 --e2e-steps 1 \
      > gpurun_out/routed_${TAG}_${cfg}_$plane.log 2>&1
  echo "$cfg $plane rc=$?" >> gpurun_out/routed_${TAG}.txt
done
echo done
