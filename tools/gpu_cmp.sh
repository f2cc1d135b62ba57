# usage (gpurun): bash tools/gpu_cmp.sh "JOBS" "VARIANTS" [tests: 1]
python tools/build.py > gpurun_out/build.log 2>&1
if [ "$3" = "1" ]; then timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1; echo rc=$? >> gpurun_out/pytest_gpu.log; fi
timeout 1200 python tools/variants.py run $1 -- $2 $2 > gpurun_out/var.jsonl 2> gpurun_out/var.err
