cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out/r2v
timeout 900 python -m pytest tests/test_gpu_convert.py tests/test_gpu_bitmap_exhaustive.py tests/test_gpu_vcycle.py -m gpu -x -q > gpurun_out/r2v/pytest.log 2>&1
echo "pytest rc=$?" >> gpurun_out/r2v/pytest.log
M=gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum
timeout 600 ncu --metrics $M --clock-control none --nvtx --nvtx-include 'setup/' --csv --log-file gpurun_out/r2v/setup.csv python tools/setup_kernels.py cfg3 > gpurun_out/r2v/setup.log 2>&1
echo done > gpurun_out/r2v/done
