cd $GRAFT_REPO_ROOT; O=gpurun_out/r2late; mkdir -p $O
timeout 900 python -m pytest tests/test_gpu_spgemm.py -x -q -m gpu > $O/t_spgemm6.log 2>&1; tail -3 $O/t_spgemm6.log
python tools/r2late/sym_var.py 2>&1 | tail -4
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -k regex:'^k_' --csv --log-file $O/cfg4_launches6.csv python tools/profile_cfg4.py 2 > $O/cfg4_ncu6.log 2>&1
python tools/ncu_sum_launches.py $O/cfg4_launches6.csv --per-launch > $O/cfg4_launches6.txt 2>&1
