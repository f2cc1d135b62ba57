# overlapped gather eviction (GROUP): parity + C4 A/B. bash tools/gpu_r11.sh TAG
TAG=${1:-r11}
mkdir -p gpurun_out
python tools/build.py > gpurun_out/build_$TAG.log 2>&1 || { echo build failed; exit 1; }
timeout 1200 python -m pytest tests/test_hot_parity_gpu.py tests/test_parity_gpu.py tests/test_fullsize_gpu.py -x -q -p no:cacheprovider -k "c4 or C4 or group or evict_overlap or placement" > gpurun_out/pytest_$TAG.log 2>&1
echo "pytest rc=$?" >> gpurun_out/pytest_$TAG.log
AB_SPECS="C4 3|C4 1" bash tools/ab.sh ov_$TAG "SEPO_EVICT_OVERLAP=0" "SEPO_EVICT_OVERLAP=1"
echo done
