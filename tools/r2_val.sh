cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out/r2val
timeout 1800 python -m pytest tests -q -m gpu -x > gpurun_out/r2val/gpu_tests.log 2>&1; echo "rc=$?" >> gpurun_out/r2val/gpu_tests.log
timeout 600 python bench.py > gpurun_out/r2val/bench.json 2> gpurun_out/r2val/bench.err
echo done > gpurun_out/r2val/done
