mkdir -p gpurun_out
python tools/build.py > gpurun_out/build_m1.log 2>&1 || exit 1
timeout 600 python -m pytest tests/test_shard_gpu.py -x -q -p no:cacheprovider -k "run_sharded" > gpurun_out/pytest_m1.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_m1.log
timeout 600 python bench.py --route --plane lib --config C5u --steps 3 --warmup 3 --e2e-steps 1 > gpurun_out/routed_m1_C5u_lib.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:insert_stream_kernel -s 1 -c 1 \
      -o gpurun_out/m1src -f python tools/time_job.py C2 0.5 > gpurun_out/ncu_m1src.log 2>&1
echo done
