# Round evidence on one GPU: bench line, ncu launch list, ncu --set full of the dominant kernels,
# residency ablation. usage (gpurun): bash tools/evidence.sh TAG
TAG=${1:-r01}
python tools/build.py > gpurun_out/build.log 2>&1
timeout 900 python bench.py > gpurun_out/bench_$TAG.log 2>&1
tail -1 gpurun_out/bench_$TAG.log > gpurun_out/bench_$TAG.json
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 600 --csv --log-file gpurun_out/launches_$TAG.csv \
    python bench.py --steps 1 --warmup 3 --no-cpu --no-curve --no-text --e2e-steps 1 > /dev/null 2>&1
timeout 900 ncu --set full --import-source on --clock-control none -k regex:insert_stream -s 1 -c 1 \
    -o gpurun_out/ins_$TAG -f python tools/time_job.py C2 4 > /dev/null 2>&1
timeout 600 ncu --set full --import-source on --clock-control none -k regex:reinsert -c 1 \
    -o gpurun_out/reins_$TAG -f python tools/time_job.py C2 4 > /dev/null 2>&1
timeout 900 python tools/ablation_residency.py --scale 1 --reps 2 --out gpurun_out/ablation_$TAG.json > gpurun_out/abl_$TAG.log 2>&1
echo done >> gpurun_out/bench_$TAG.log
