# GROUP eviction overlap: parity + C4 timing A/B. bash tools/gpu_r10.sh TAG
TAG=${1:-r10}
mkdir -p gpurun_out
python tools/build.py > gpurun_out/build_$TAG.log 2>&1 || { echo build failed; exit 1; }
timeout 900 python -m pytest tests/test_hot_parity_gpu.py -x -q -p no:cacheprovider -k "evict_overlap or c4" > gpurun_out/pytest_$TAG.log 2>&1
echo "pytest rc=$?" >> gpurun_out/pytest_$TAG.log
AB_SPECS="C4 3" bash tools/ab.sh ov_$TAG "SEPO_EVICT_OVERLAP=0" "SEPO_EVICT_OVERLAP=1"
echo done
