cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out/r2
timeout 900 python -m pytest tests/test_gpu_convert.py tests/test_gpu_spgemm.py tests/test_gpu_pmis.py -q -m gpu -x > gpurun_out/r2/conv_tests.log 2>&1; echo "rc=$?" >> gpurun_out/r2/conv_tests.log
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --nvtx --nvtx-include 'setup/' --csv --log-file gpurun_out/r2/setup_cfg3_launches_c.csv python tools/setup_kernels.py cfg3 > gpurun_out/r2/setup_cfg3.log 2>&1
