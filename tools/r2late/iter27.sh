cd $GRAFT_REPO_ROOT
timeout 1500 python -m pytest tests -x -q -m gpu 2>&1 | tail -1
for v in "AMGT_SPGEMM_DET=1" "AMGT_SPGEMM_DET=0"; do
env $v python -c "
import sys, json; sys.path.insert(0, '.')
import torch, bench, paper_conf_sc_luzwflcy0c024_b200 as amgt
print('$v', json.dumps({k: v for k, v in bench.spgemm_cfg4(amgt, torch, 6539.2).items() if k in ('ms', 'symbolic_ms', 'numeric_ms')}))
" 2>&1 | tail -1
done
AMGT_SPGEMM_DET=1 python tools/r2late/symvar_mem.py 0 2>&1 | tail -3
