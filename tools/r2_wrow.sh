cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out/r2h
timeout 900 python -m pytest tests/test_gpu_vcycle.py tests/test_gpu_dist.py tests/test_gpu_spmv.py tests/test_gpu_full.py tests/test_gpu_pcg.py -m gpu -x -q > gpurun_out/r2h/pytest.log 2>&1
echo "pytest rc=$?" >> gpurun_out/r2h/pytest.log
M=gpu__time_duration.sum,dram__bytes_read.sum
for v in 65536 10000000 0; do
AMGT_SPMV_WROW=$v timeout 600 ncu --metrics $M --clock-control none --kernel-name-base demangled -k regex:'k_spmv_(rows|wrow)<(float|__half)' --csv --log-file gpurun_out/r2h/l_$v.csv python tools/profile_vcycle.py 2 cfg3 > /dev/null 2>&1
AMGT_SPMV_WROW=$v timeout 300 python bench.py --steps 5 --warmup 3 --no-cpu-baseline --no-cfg4 > gpurun_out/r2h/bench_$v.json 2>/dev/null
done
echo done > gpurun_out/r2h/done
