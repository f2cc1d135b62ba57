# router determinism tests, head-hint parity + A/B, routed trace. bash tools/gpu_r5.sh TAG
TAG=${1:-r5}
mkdir -p gpurun_out
python tools/build.py > gpurun_out/build_$TAG.log 2>&1 || { echo build failed; exit 1; }
timeout 900 python -m pytest tests/test_shard_gpu.py tests/test_hot_parity_gpu.py -x -q -p no:cacheprovider > gpurun_out/pytest_$TAG.log 2>&1
echo "pytest rc=$?" >> gpurun_out/pytest_$TAG.log
python tools/variants.py run C2:0.5 C2:4 C3:1 C5u:4 -- base hint0 base+SEPO_LEAN=1 > gpurun_out/var_$TAG.jsonl 2>&1
SEPO_TRACE=1 timeout 600 python bench.py --route --plane lib --config C5z --steps 1 --warmup 3 --e2e-steps 0 > gpurun_out/trace_${TAG}_C5z.log 2>&1
for r in C2:torch C5z:torch; do
  cfg=${r%%:*}; plane=${r##*:}
  timeout 600 python bench.py --route --plane $plane --config $cfg --steps 5 --warmup 3 --e2e-steps 1 \
      > gpurun_out/routed_${TAG}_${r/:/_}.log 2>&1
  echo "$r rc=$?" >> gpurun_out/routed_${TAG}.txt
done
echo done
