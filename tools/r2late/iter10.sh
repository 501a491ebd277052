cd $GRAFT_REPO_ROOT; O=gpurun_out/r2late; mkdir -p $O
timeout 900 python -m pytest tests/test_gpu_spgemm.py -x -q -m gpu > $O/t10.log 2>&1; tail -2 $O/t10.log
python tools/r2late/sym_var.py 2>&1 | tail -3
