cd $GRAFT_REPO_ROOT; O=gpurun_out/r2late; mkdir -p $O
timeout 1500 python -m pytest tests -x -q -m gpu > $O/gpu_all3.log 2>&1; tail -3 $O/gpu_all3.log
python tools/r2late/sym_var.py 2>&1 | tail -2
python tools/r2late/setup_time.py cfg3 3 2>&1 | tail -1
