# A*P one-tile-row numeric fast path: parity tests, then cfg3 setup launch lists with / without it,
# then the 512^3 virtual-rank overhead sweep (G=1,2,4,8 in one process)
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out/r2b
timeout 1200 python -m pytest tests/test_gpu_spgemm.py tests/test_gpu_vcycle.py tests/test_gpu_interp.py tests/test_gpu_dist.py tests/test_gpu_pmis.py -m gpu -x -q > gpurun_out/r2b/pytest.log 2>&1
echo "pytest rc=$?" >> gpurun_out/r2b/pytest.log
M=gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum
timeout 600 ncu --metrics $M --clock-control none --nvtx --nvtx-include 'setup/' --csv --log-file gpurun_out/r2b/setup_b1.csv python tools/setup_kernels.py cfg3 > gpurun_out/r2b/setup_b1.log 2>&1
AMGT_NUM_B1=0 timeout 600 ncu --metrics $M --clock-control none --nvtx --nvtx-include 'setup/' --csv --log-file gpurun_out/r2b/setup_nob1.csv python tools/setup_kernels.py cfg3 > gpurun_out/r2b/setup_nob1.log 2>&1
timeout 300 python bench.py --steps 5 --warmup 3 --no-cpu-baseline --no-cfg4 > gpurun_out/r2b/bench_b1.json 2> gpurun_out/r2b/bench_b1.err
AMGT_NUM_B1=0 timeout 300 python bench.py --steps 5 --warmup 3 --no-cpu-baseline --no-cfg4 > gpurun_out/r2b/bench_nob1.json 2> gpurun_out/r2b/bench_nob1.err
timeout 1500 python tools/dist_overhead.py --n 512 --cycles 10 --agg-rows 262144 > gpurun_out/r2b/dist_overhead_512.jsonl 2> gpurun_out/r2b/dist_overhead_512.err
echo done > gpurun_out/r2b/done
