# ncu --set full of the raw-text pass-1 kernel: bash tools/ncu_text.sh NAME KREGEX RATIO [ENV...]
NAME=$1; K=$2; R=$3; shift 3
python tools/build.py > gpurun_out/build_$NAME.log 2>&1 || exit 1
env "$@" timeout 900 ncu --set full --clock-control none --import-source on -k regex:$K -s 1 -c 1 -o gpurun_out/$NAME -f \
    python tools/time_text.py $R > gpurun_out/ncu_$NAME.log 2>&1
echo rc=$? >> gpurun_out/ncu_$NAME.log
