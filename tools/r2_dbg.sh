cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out/r2
timeout 1200 python tools/table2_run.py > gpurun_out/r2/table2.jsonl 2> gpurun_out/r2/table2.err
