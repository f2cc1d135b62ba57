# round-2 evidence session (M1 = insert_lean_kernel since the in-budget CSR switch): tests, ncu captures of the kernels the bench line reports, the launch list, the bench
TAG=${1:-r02}
python tools/build.py > gpurun_out/build_$TAG.log 2>&1 || exit 1
if [ "${SKIP_TESTS:-0}" != 1 ]; then
  timeout 1500 python -m pytest -x -q -p no:cacheprovider tests -m gpu > gpurun_out/pytest_$TAG.log 2>&1; echo rc=$? >> gpurun_out/pytest_$TAG.log
  timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke_$TAG.log 2>&1
fi
if [ "${SKIP_NCU:-0}" != 1 ]; then
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:insert_lean_kernel -s 1 -c 1 \
      -o gpurun_out/m1_$TAG -f python tools/time_job.py C2 0.5 > gpurun_out/ncu_m1_$TAG.log 2>&1
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:insert_text2 -s 1 -c 1 \
      -o gpurun_out/text_$TAG -f python tools/time_text.py 4 > gpurun_out/ncu_text_$TAG.log 2>&1
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:insert_stream_kernel -s 1 -c 1 \
      -o gpurun_out/c3_$TAG -f python tools/time_job.py C3 1 > gpurun_out/ncu_c3_$TAG.log 2>&1
  timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_$TAG.csv \
      python bench.py --steps 2 --warmup 1 --no-curve --e2e-steps 0 --no-cpu --no-m1-c3 > gpurun_out/launches_$TAG.log 2>&1
fi
if [ "${SKIP_BENCH:-0}" != 1 ]; then
  timeout 900 python bench.py > gpurun_out/bench_$TAG.log 2>&1
  tail -1 gpurun_out/bench_$TAG.log > gpurun_out/bench_$TAG.json
fi
echo done
