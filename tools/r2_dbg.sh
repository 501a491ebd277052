cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out/r2
timeout 900 python -m pytest tests/test_gpu_pmis.py -q -m gpu > gpurun_out/r2/pmis_tests.log 2>&1; echo "rc=$?" >> gpurun_out/r2/pmis_tests.log
timeout 900 ncu --set full --clock-control none --kernel-name-base demangled -k regex:'k_spmv_rows<double, double, double' -c 4 -f -o gpurun_out/r2/ncu_spmv_cfg3 python tools/ncu_traffic.py run cfg3 > gpurun_out/r2/ncu_cfg3.log 2>&1
