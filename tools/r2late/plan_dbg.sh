cd $GRAFT_REPO_ROOT
python tools/r2late/plan_dbg.py; AMGT_SPGEMM_PLAN=0 python tools/r2late/plan_dbg.py
