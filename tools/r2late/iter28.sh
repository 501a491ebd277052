cd $GRAFT_REPO_ROOT; O=gpurun_out/r2late; mkdir -p $O
timeout 1200 python -m pytest tests/test_gpu_spgemm.py tests/test_gpu_vcycle.py -x -q -m gpu 2>&1 | tail -1
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --nvtx --nvtx-include 'setup/' -k regex:'^k_numeric$' --csv --log-file $O/knum3.csv python tools/setup_kernels.py cfg3 > /dev/null 2>&1
python tools/ncu_sum_launches.py $O/knum3.csv | head -3
python tools/r2late/sym_var.py 2>&1 | tail -1
