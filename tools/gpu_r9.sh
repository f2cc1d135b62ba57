# lean hot-sum atomic + full-size sharded closed forms. bash tools/gpu_r9.sh TAG
TAG=${1:-r9}
mkdir -p gpurun_out
python tools/build.py > gpurun_out/build_$TAG.log 2>&1 || { echo build failed; exit 1; }
timeout 300 python tools/time_job.py C2 0.5 > gpurun_out/m1_$TAG.json 2>&1
timeout 300 python tools/time_job.py C2 4 > gpurun_out/c2x4_$TAG.json 2>&1
timeout 1200 python -m pytest tests/test_fullsize_gpu.py tests/test_hot_parity_gpu.py -x -q -p no:cacheprovider > gpurun_out/pytest_$TAG.log 2>&1
echo "pytest rc=$?" >> gpurun_out/pytest_$TAG.log
echo done
