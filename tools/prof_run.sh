# usage: bash tools/prof_run.sh NAME CFG RATIO [LIB]
python tools/build.py > gpurun_out/build.log 2>&1
export SEPO_LIB=${4:-paper_conf_ipps_mokhtaris17_b200/lib/libsepo.so}
timeout 900 ncu --set full --clock-control none --import-source on -k regex:insert_stream -c 1 -o gpurun_out/$1 -f python tools/time_job.py $2 $3 > gpurun_out/$1.log 2>&1
echo rc=$? >> gpurun_out/$1.log
