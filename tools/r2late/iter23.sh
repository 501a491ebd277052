cd $GRAFT_REPO_ROOT
AMGT_SCRATCH_CACHE_MB=32768 python tools/r2late/sym_var.py 2>&1 | tail -5
AMGT_SPGEMM_DET=0 python tools/r2late/sym_var.py 2>&1 | tail -3
