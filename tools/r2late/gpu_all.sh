cd $GRAFT_REPO_ROOT; O=gpurun_out/r2late; mkdir -p $O
timeout 2400 python -m pytest tests -x -q -m gpu > $O/gpu_all.log 2>&1; tail -5 $O/gpu_all.log
python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke.log 2>&1; tail -2 $O/smoke.log
