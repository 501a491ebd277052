cd $GRAFT_REPO_ROOT; O=gpurun_out/r2late; mkdir -p $O
timeout 1200 python -m pytest tests/test_gpu_spgemm.py -x -q -m gpu > $O/t21.log 2>&1; tail -4 $O/t21.log
python tools/r2late/sym_var.py 2>&1 | tail -2
AMGT_SPGEMM_DET=0 python tools/r2late/sym_var.py 2>&1 | tail -1
