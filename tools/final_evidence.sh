# Full round evidence on one GPU: every GPU test, smoke, bench line, ncu launch list of the bench
# command, ncu --set full of the pass-1 insert kernel. usage (gpurun): bash tools/final_evidence.sh TAG
TAG=${1:-r01}
python tools/build.py > gpurun_out/build.log 2>&1
timeout 1500 python -m pytest tests -m gpu -q > gpurun_out/pytest_gpu_$TAG.log 2>&1; echo rc=$? >> gpurun_out/pytest_gpu_$TAG.log
timeout 300 python __graft_entry__.py smoke > gpurun_out/smoke_$TAG.log 2>&1; echo rc=$? >> gpurun_out/smoke_$TAG.log
timeout 900 python bench.py > gpurun_out/bench_$TAG.log 2>&1
tail -1 gpurun_out/bench_$TAG.log > gpurun_out/bench_$TAG.json
timeout 900 python bench.py --impl reference --steps 2 --warmup 1 > gpurun_out/bench_ref_$TAG.log 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 600 --csv --log-file gpurun_out/launches_$TAG.csv \
    python bench.py --steps 1 --warmup 3 --no-cpu --no-curve --no-text --e2e-steps 1 > /dev/null 2>&1
timeout 900 ncu --set full --import-source on --clock-control none -k regex:insert_stream -s 1 -c 1 \
    -o gpurun_out/ins_$TAG -f python tools/time_job.py C2 4 > /dev/null 2>&1
echo done >> gpurun_out/bench_$TAG.log
