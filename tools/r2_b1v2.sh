# A*P one-tile-row numeric (metadata-first chunks, shared-memory accumulators): parity + setup launch list + ncu full
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out/r2c
timeout 1200 python -m pytest tests/test_gpu_spgemm.py tests/test_gpu_vcycle.py tests/test_gpu_interp.py tests/test_gpu_pmis.py tests/test_gpu_dist.py tests/test_gpu_full.py -m gpu -x -q > gpurun_out/r2c/pytest.log 2>&1
echo "pytest rc=$?" >> gpurun_out/r2c/pytest.log
M=gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum
timeout 600 ncu --metrics $M --clock-control none --nvtx --nvtx-include 'setup/' --csv --log-file gpurun_out/r2c/setup_b1.csv python tools/setup_kernels.py cfg3 > gpurun_out/r2c/setup_b1.log 2>&1
timeout 900 ncu --set full --import-source on --clock-control none --nvtx --nvtx-include 'setup/' -k regex:k_numeric_b1 -c 1 -o gpurun_out/r2c/b1_full python tools/setup_kernels.py cfg3 > gpurun_out/r2c/b1_full.log 2>&1
echo done > gpurun_out/r2c/done
