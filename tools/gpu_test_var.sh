python tools/build.py > gpurun_out/build.log 2>&1
timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1; echo rc=$? >> gpurun_out/pytest_gpu.log
timeout 900 python tools/variants.py run $1 -- $2 > gpurun_out/var.jsonl 2> gpurun_out/var.err
