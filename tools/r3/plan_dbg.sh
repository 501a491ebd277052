cd $GRAFT_REPO_ROOT
python tools/r3/plan_dbg.py; AMGT_SPGEMM_PLAN=0 python tools/r3/plan_dbg.py
