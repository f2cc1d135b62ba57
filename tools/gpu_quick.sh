# usage: bash tools/gpu_quick.sh "JOBS" "VARIANTS" [gpu tests: 1]
python tools/build.py > gpurun_out/build.log 2>&1
if [ "$3" = "1" ]; then timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1; echo rc=$? >> gpurun_out/pytest_gpu.log; fi
timeout 900 python tools/variants.py run $1 -- $2 > gpurun_out/var.jsonl 2> gpurun_out/var.err
for v in $2; do
  SEPO_LIB=exp/lib_$v.so timeout 300 ncu --metrics dram__bytes_read.sum,gpu__time_duration.sum,smsp__inst_executed.sum,smsp__issue_active.avg.pct_of_peak_sustained_active --clock-control none -k regex:insert_stream -c 1 --csv python tools/time_job.py C2 0.5 > gpurun_out/ncuq_$v.csv 2>&1
done
