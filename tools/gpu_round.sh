# One GPU session of round 2 (gpurun): tests, the bench line, the launch list and ncu captures.
#   bash tools/gpu_round.sh TAG [tests|bench|ncu|all]...
TAG=${1:-r2}; shift
WHAT=${@:-all}
mkdir -p gpurun_out
python tools/build.py > gpurun_out/build_$TAG.log 2>&1 || { echo build failed; exit 1; }
has() { [[ " $WHAT " == *" $1 "* || " $WHAT " == *" all "* ]]; }
if has tests; then
  timeout 1500 python -m pytest tests -m gpu -x -q -p no:cacheprovider > gpurun_out/pytest_$TAG.log 2>&1
  echo "pytest rc=$?" >> gpurun_out/pytest_$TAG.log
  timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke_$TAG.log 2>&1
fi
if has bench; then
  timeout 900 python bench.py > gpurun_out/bench_$TAG.log 2>&1
  tail -1 gpurun_out/bench_$TAG.log > gpurun_out/bench_$TAG.json
fi
if has ncu; then
  # M1 kernel: pass 1 of the in-budget C2 job (0.5x); headline kernel: pass 1 of the raw-text job (4x)
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:insert_stream_kernel -s 1 -c 1 \
      -o gpurun_out/m1_$TAG -f python tools/time_job.py C2 0.5 > gpurun_out/ncu_m1_$TAG.log 2>&1
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:insert_text_kernel -s 1 -c 1 \
      -o gpurun_out/text_$TAG -f python tools/time_text.py 4 > gpurun_out/ncu_text_$TAG.log 2>&1
  timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_$TAG.csv \
      python bench.py --steps 2 --warmup 1 --no-curve --e2e-steps 0 --no-cpu --no-m1-c3 > gpurun_out/launches_$TAG.log 2>&1
fi
if has c3; then
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:insert_stream_kernel -s 1 -c 1 \
      -o gpurun_out/c3_$TAG -f python tools/time_job.py C3 1 > gpurun_out/ncu_c3_$TAG.log 2>&1
fi
if has c4; then
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:insert_group_stream -s 1 -c 1 \
      -o gpurun_out/c4_$TAG -f python tools/time_job.py C4 3 > gpurun_out/ncu_c4_$TAG.log 2>&1
fi
if has configs; then
  bash tools/bench_configs.sh $TAG
fi
echo done
