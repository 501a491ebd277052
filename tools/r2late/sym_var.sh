cd $GRAFT_REPO_ROOT
python tools/r2late/sym_var.py; echo "--- cache 16G"; AMGT_SCRATCH_CACHE_MB=16384 python tools/r2late/sym_var.py
echo "--- dense 3"; AMGT_DENSE_FROM_BIN=3 AMGT_SCRATCH_CACHE_MB=16384 python tools/r2late/sym_var.py
echo "--- dense 4"; AMGT_DENSE_FROM_BIN=4 AMGT_SCRATCH_CACHE_MB=16384 python tools/r2late/sym_var.py
