# GROUP overlapped gather fix: C4 full-size closed forms repeatedly + GROUP parity + timing
mkdir -p gpurun_out
python tools/build.py > gpurun_out/build_r14.log 2>&1 || { echo build failed; exit 1; }
timeout 1500 python -m pytest tests/test_fullsize_gpu.py tests/test_hot_parity_gpu.py -q -p no:cacheprovider -k "c4 or C4 or evict_overlap" > gpurun_out/pytest_r14a.log 2>&1; echo rc=$? >> gpurun_out/pytest_r14a.log
for i in 1 2 3 4; do timeout 600 python -m pytest tests/test_fullsize_gpu.py -q -p no:cacheprovider -k "c4_full" > gpurun_out/pytest_r14_c4_$i.log 2>&1; echo rc=$? >> gpurun_out/pytest_r14_c4_$i.log; done
timeout 300 python tools/time_job.py C4 3 > gpurun_out/time_r14_C4.json 2>&1
echo done
