# final evidence after the GROUP overlap / vectorised scatter changes. bash tools/gpu_final3.sh TAG
TAG=${1:-r02f}
mkdir -p gpurun_out
python tools/build.py > gpurun_out/build_$TAG.log 2>&1 || { echo build failed; exit 1; }
timeout 1800 python -m pytest -x -q -p no:cacheprovider tests -m gpu > gpurun_out/pytest_$TAG.log 2>&1; echo rc=$? >> gpurun_out/pytest_$TAG.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke_$TAG.log 2>&1
timeout 900 python bench.py > gpurun_out/bench_$TAG.log 2>&1
tail -1 gpurun_out/bench_$TAG.log > gpurun_out/bench_$TAG.json
timeout 600 python bench.py --impl reference --steps 2 --warmup 1 > gpurun_out/ref_$TAG.log 2>&1
tail -1 gpurun_out/ref_$TAG.log > gpurun_out/ref_$TAG.json
for c in C4 C5u C3; do timeout 600 python tools/time_job.py $c $( [ $c = C4 ] && echo 3 || echo 4 ) $( [ $c = C5u ] && echo 0.125 ) > gpurun_out/cfg_${TAG}_$c.json 2>&1; done
echo done
