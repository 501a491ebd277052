cd $GRAFT_REPO_ROOT; O=gpurun_out/r2late; mkdir -p $O
timeout 1200 python -m pytest tests/test_gpu_spgemm.py tests/test_gpu_vcycle.py -x -q -m gpu > $O/t17.log 2>&1; tail -3 $O/t17.log
python tools/r2late/sym_var.py 2>&1 | tail -2
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:'^k_' --csv --log-file $O/l17.csv python tools/profile_cfg4.py 2 > /dev/null 2>&1
python tools/ncu_sum_launches.py $O/l17.csv --per-launch 2>&1 | awk '$1>=52' | head -30
