# vectorised CSR scatter: router tests + routed C3. bash tools/gpu_r12.sh TAG
TAG=${1:-r12}
mkdir -p gpurun_out
python tools/build.py > gpurun_out/build_$TAG.log 2>&1 || { echo build failed; exit 1; }
timeout 900 python -m pytest tests/test_shard_gpu.py -x -q -p no:cacheprovider > gpurun_out/pytest_$TAG.log 2>&1
echo "pytest rc=$?" >> gpurun_out/pytest_$TAG.log
timeout 600 python bench.py --route --config C3 --steps 5 --warmup 3 --e2e-steps 1 > gpurun_out/routed_${TAG}_C3.log 2>&1
SEPO_SHARD_WIRE=0 timeout 600 python bench.py --route --config C2 --steps 5 --warmup 3 --e2e-steps 1 --plane lib > gpurun_out/routed_${TAG}_C2csr.log 2>&1 </dev/null
echo done
