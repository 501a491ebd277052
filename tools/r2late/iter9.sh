cd $GRAFT_REPO_ROOT; O=gpurun_out/r2late; mkdir -p $O
timeout 900 python -m pytest tests/test_gpu_spgemm.py tests/test_gpu_vcycle.py -x -q -m gpu > $O/t9.log 2>&1; tail -2 $O/t9.log
python tools/r2late/sym_var.py 2>&1 | tail -2
python tools/r2late/setup_time.py cfg3 3 2>&1 | tail -1
