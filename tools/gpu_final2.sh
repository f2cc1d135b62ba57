# final round-2 evidence: GPU tests + smoke, ncu of the M1 kernel, bench launch list, bench line,
# routed lines at N = 1. bash tools/gpu_final2.sh TAG
TAG=${1:-r02e}
mkdir -p gpurun_out
python tools/build.py > gpurun_out/build_$TAG.log 2>&1 || { echo build failed; exit 1; }
timeout 1800 python -m pytest -x -q -p no:cacheprovider tests -m gpu > gpurun_out/pytest_$TAG.log 2>&1; echo rc=$? >> gpurun_out/pytest_$TAG.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke_$TAG.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:insert_lean_kernel -s 1 -c 1 \
    -o gpurun_out/m1_$TAG -f python tools/time_job.py C2 0.5 > gpurun_out/ncu_m1_$TAG.log 2>&1
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_$TAG.csv \
    python bench.py --steps 2 --warmup 1 --no-curve --e2e-steps 0 --no-cpu --no-m1-c3 > gpurun_out/launches_$TAG.log 2>&1
timeout 900 python bench.py > gpurun_out/bench_$TAG.log 2>&1
tail -1 gpurun_out/bench_$TAG.log > gpurun_out/bench_$TAG.json
for r in C2 C5z C5u; do
  timeout 600 python bench.py --route --config $r --steps 5 --warmup 3 --e2e-steps 1 > gpurun_out/routed_${TAG}_$r.log 2>&1
  echo "$r rc=$?" >> gpurun_out/routed_${TAG}.txt
done
echo done
