cd $GRAFT_REPO_ROOT; O=gpurun_out/r3; mkdir -p $O
timeout 1500 python -m pytest tests -x -q -m gpu > $O/gpu_all3.log 2>&1; tail -3 $O/gpu_all3.log
python tools/r3/sym_var.py 2>&1 | tail -2
python tools/r3/setup_time.py cfg3 3 2>&1 | tail -1
