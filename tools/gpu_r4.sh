# router tests, routed lines, M1 knob A/B. bash tools/gpu_r4.sh TAG
TAG=${1:-r4}
mkdir -p gpurun_out
python tools/build.py > gpurun_out/build_$TAG.log 2>&1 || { echo build failed; exit 1; }
timeout 900 python -m pytest tests/test_shard_gpu.py -x -q -p no:cacheprovider > gpurun_out/pytest_$TAG.log 2>&1
echo "pytest rc=$?" >> gpurun_out/pytest_$TAG.log
for r in C2:lib C2:torch C5z:lib C5z:torch C3:lib; do
  cfg=${r%%:*}; plane=${r##*:}
  timeout 600 python bench.py --route --plane $plane --config $cfg --steps 5 --warmup 3 --e2e-steps 1 \
      > gpurun_out/routed_${TAG}_${r/:/_}.log 2>&1
  echo "$r rc=$?" >> gpurun_out/routed_${TAG}.txt
done
AB_SPECS="C2 0.5" bash tools/ab.sh m1_$TAG "SEPO_LEAN=0" "SEPO_LEAN=1" "SEPO_DIR_PF=0"
echo done
