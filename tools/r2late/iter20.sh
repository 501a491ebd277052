cd $GRAFT_REPO_ROOT; O=gpurun_out/r2late; mkdir -p $O
timeout 1200 python -m pytest tests/test_gpu_spgemm.py -x -q -m gpu > $O/t20.log 2>&1; tail -2 $O/t20.log
python tools/r2late/sym_var.py 2>&1 | tail -2
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:'k_sym' --csv --log-file $O/l20.csv python tools/profile_cfg4.py 2 > /dev/null 2>&1
python tools/ncu_sum_launches.py $O/l20.csv 2>&1 | head -6
