cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out/r2
for i in 1 2 3; do timeout 600 python -m pytest tests/test_gpu_dist.py -q -m gpu -x > gpurun_out/r2/t$i.log 2>&1; done
