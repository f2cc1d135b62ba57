# A/B: hot-key value fold (warp fold vs per-hit shared atomics). bash tools/gpu_r13.sh
mkdir -p gpurun_out
python tools/variants.py run C5z:4:0.125 C5u:4:0.125 -- base fold1 base fold1 > gpurun_out/var_fold.jsonl 2>&1
for v in base fold1; do
  SEPO_LIB=exp/lib_$v.so timeout 600 python bench.py --route --config C5z --steps 5 --warmup 3 --e2e-steps 0 > gpurun_out/routed_fold_$v.log 2>&1
done
SEPO_LIB=exp/lib_fold1.so timeout 900 python -m pytest tests/test_shard_gpu.py tests/test_hot_parity_gpu.py -x -q -p no:cacheprovider -k "c5 or C5 or route" > gpurun_out/pytest_fold1.log 2>&1; echo rc=$? >> gpurun_out/pytest_fold1.log
echo done
