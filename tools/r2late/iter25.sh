cd $GRAFT_REPO_ROOT
for v in "X=1" "AMGT_SPGEMM_PLAN=0" "AMGT_SCRATCH_CACHE_MB=0" "AMGT_SCRATCH_CACHE_MB=65536" "AMGT_GDENSE=0"; do
env $v python -c "
import sys, json; sys.path.insert(0, '.')
import torch, bench, paper_conf_sc_luzwflcy0c024_b200 as amgt
print('$v', json.dumps({k: v for k, v in bench.spgemm_cfg4(amgt, torch, 6539.2).items() if k in ('ms', 'symbolic_ms', 'numeric_ms')}))
" 2>&1 | tail -1
done
