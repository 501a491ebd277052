cd $GRAFT_REPO_ROOT; O=gpurun_out/r2late; mkdir -p $O
timeout 900 python -m pytest tests/test_gpu_spgemm.py -x -q -m gpu > $O/t14.log 2>&1; tail -2 $O/t14.log
for v in 0 1; do echo "WARP=$v"; AMGT_PLAN_WARP=$v python tools/r2late/sym_var.py 2>&1 | tail -2; done
