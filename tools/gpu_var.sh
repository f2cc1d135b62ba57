# usage (on the GPU box): bash tools/gpu_var.sh "JOBS" "VARIANTS" [ncu_variant]
python tools/build.py > gpurun_out/build.log 2>&1
timeout 900 python tools/variants.py run $1 -- $2 > gpurun_out/var.jsonl 2> gpurun_out/var.err
if [ -n "$3" ]; then
  for v in $3; do
  SEPO_LIB=exp/lib_$v.so timeout 300 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum,lts__t_sector_hit_rate.pct,smsp__inst_executed.sum --clock-control none -k regex:insert_stream -c 5 --csv python tools/time_job.py C2 4 > gpurun_out/ncu_$v.csv 2>&1
  done
fi
