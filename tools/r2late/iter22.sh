cd $GRAFT_REPO_ROOT; O=gpurun_out/r2late; mkdir -p $O
python tools/r2late/sym_var.py 2>&1 | tail -8
AMGT_TRACE=1 python tools/r2late/sym_var.py 2>&1 | grep trace | tail -12
