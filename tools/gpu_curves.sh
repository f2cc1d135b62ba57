# M3 slowdown curves for C3, C4, C5u, C5z + the oversubscribed managed-pool ablation
TAG=${1:-r2}
python tools/build.py > gpurun_out/build_$TAG.log 2>&1 || exit 1
: > gpurun_out/curves_$TAG.jsonl
for spec in "C3 4 1" "C4 3 1" "C5u 4 0.125" "C5z 4 0.125"; do
  set -- $spec
  timeout 900 python bench.py --config $1 --ratio $2 --scale $3 --steps 3 --warmup 3 --no-cpu --no-m1 --no-m1-c3 --e2e-steps 0 \
      > gpurun_out/curve_$1.log 2>&1
  tail -1 gpurun_out/curve_$1.log >> gpurun_out/curves_$TAG.jsonl
done
timeout 900 python tools/ablation_residency.py --scale 0.0625 --reps 2 --out gpurun_out/ablation_oversub_$TAG.json \
    > gpurun_out/ablation_oversub_$TAG.log 2>&1
echo done
