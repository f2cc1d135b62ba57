# One bench line per BASELINE config (context for SURVEY §8(d) M1-M3; the headline is C2 at 4x).
# usage (gpurun): bash tools/bench_configs.sh TAG
TAG=${1:-cfg}
python tools/build.py > gpurun_out/build.log 2>&1
: > gpurun_out/configs_$TAG.jsonl
for spec in "C1 1 1" "C1 4 1" "C3 1 1" "C3 4 1" "C4 3 1" "C5u 4 0.125" "C5z 4 0.125" "C2 0.5 1" "C2 1 1" "C2 2 1"; do
  set -- $spec
  timeout 900 python bench.py --config $1 --ratio $2 --scale $3 --steps 3 --warmup 3 --no-cpu --no-curve --e2e-steps 0 \
      > gpurun_out/cfg_$1_$2.log 2>&1
  tail -1 gpurun_out/cfg_$1_$2.log >> gpurun_out/configs_$TAG.jsonl
done
