# C4 (GROUP) breakdown: phase times at full size, kernel launch list at 1/4. bash tools/gpu_c4.sh TAG
TAG=${1:-c4}
mkdir -p gpurun_out
python tools/build.py > gpurun_out/build_$TAG.log 2>&1 || { echo build failed; exit 1; }
timeout 600 python tools/time_job.py C4 3 > gpurun_out/time_${TAG}_C4.json 2>&1
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_${TAG}_C4.csv \
   python tools/time_job.py C4 3 0.25 > gpurun_out/ncu_${TAG}.log 2>&1
echo done
