# GPU check of the distributed ABI (loopback virtual ranks) + the new bench line
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out/r2
python __graft_entry__.py build > gpurun_out/r2/build.log 2>&1
timeout 900 python -m pytest tests/test_gpu_dist.py -x -q -m gpu > gpurun_out/r2/dist_tests.log 2>&1
echo "dist tests rc=$?" >> gpurun_out/r2/dist_tests.log
timeout 900 python bench.py --steps 5 --warmup 3 > gpurun_out/r2/bench_cfg3.json 2> gpurun_out/r2/bench_cfg3.err
echo "bench rc=$?" >> gpurun_out/r2/bench_cfg3.err
tail -3 gpurun_out/r2/dist_tests.log gpurun_out/r2/bench_cfg3.err
