cd $GRAFT_REPO_ROOT
python tools/r2late/symvar_mem.py 0 2>&1 | tail -3
python tools/r2late/symvar_mem.py 100 2>&1 | tail -3
python -c "
import sys, json; sys.path.insert(0, '.')
import torch, bench, paper_conf_sc_luzwflcy0c024_b200 as amgt
print(json.dumps({k: v for k, v in bench.spgemm_cfg4(amgt, torch, 6539.2).items() if k in ('ms', 'symbolic_ms', 'numeric_ms')}))
" 2>&1 | tail -1
