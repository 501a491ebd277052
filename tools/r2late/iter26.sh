cd $GRAFT_REPO_ROOT
timeout 1200 python -m pytest tests/test_gpu_spgemm.py tests/test_gpu_dist.py -x -q -m gpu 2>&1 | tail -1
for v in "X=1" "X=2" "AMGT_SPGEMM_PLAN=0"; do
env $v python -c "
import sys, json; sys.path.insert(0, '.')
import torch, bench, paper_conf_sc_luzwflcy0c024_b200 as amgt
print('$v', json.dumps({k: v for k, v in bench.spgemm_cfg4(amgt, torch, 6539.2).items() if k in ('ms', 'symbolic_ms', 'numeric_ms')}))
" 2>&1 | tail -1
done
python tools/r2late/symvar_mem.py 0 2>&1 | tail -4
