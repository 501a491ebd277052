cd $GRAFT_REPO_ROOT; O=gpurun_out/r2late; mkdir -p $O
timeout 1200 python -m pytest tests/test_gpu_spgemm.py tests/test_gpu_dist.py -x -q -m gpu > $O/t16.log 2>&1; tail -3 $O/t16.log
python tools/r2late/sym_var.py 2>&1 | tail -2
