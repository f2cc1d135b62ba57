# ncu --set full of one kernel in one job: bash tools/ncu_one.sh NAME KERNEL_REGEX CFG RATIO [SCALE] [ENV...]
NAME=$1; K=$2; CFG=$3; R=$4; SC=${5:-1}; shift 5
python tools/build.py > gpurun_out/build_$NAME.log 2>&1 || exit 1
env "$@" timeout 900 ncu --set full --clock-control none --import-source on -k regex:$K -s 1 -c 1 -o gpurun_out/$NAME -f \
    python tools/time_job.py $CFG $R $SC > gpurun_out/ncu_$NAME.log 2>&1
echo rc=$? >> gpurun_out/ncu_$NAME.log
