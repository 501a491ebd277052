cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out/r2
timeout 900 python -m pytest tests/test_gpu_spmv.py -q -m gpu -x > gpurun_out/r2/spmv_tests.log 2>&1; echo "rc=$?" >> gpurun_out/r2/spmv_tests.log
timeout 600 python tools/tc_compare.py 10 spmv > gpurun_out/r2/tc_compare_spmv.json 2> gpurun_out/r2/tc_compare.err
timeout 900 ncu --set full --clock-control none -k regex:'k_spmv' -f -o gpurun_out/r2/ncu_tc_spmv python tools/tc_pipe_spmv.py > gpurun_out/r2/ncu_tc_spmv.log 2>&1
