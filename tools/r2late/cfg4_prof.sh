# cfg4 A*A: event timing, then a launch list with DRAM bytes of the second (non-info) call
cd $GRAFT_REPO_ROOT; O=gpurun_out/r2late; mkdir -p $O
python tools/spgemm_time.py cfg4 5 > $O/cfg4_time.json 2> $O/cfg4_time.err
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -k regex:'^k_' --csv --log-file $O/cfg4_launches.csv python tools/profile_cfg4.py 2 > $O/cfg4_ncu.log 2>&1
python tools/ncu_sum_launches.py $O/cfg4_launches.csv --per-launch > $O/cfg4_launches.txt 2>&1
