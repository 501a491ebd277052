cd $GRAFT_REPO_ROOT; O=gpurun_out/r2late; mkdir -p $O
timeout 900 python -m pytest tests/test_gpu_spgemm.py -x -q -m gpu > $O/t_spgemm2.log 2>&1; tail -15 $O/t_spgemm2.log
rm -f $O/cfg4_knobs2.txt
for v in "AMGT_SPGEMM_PLAN=0" "AMGT_SPGEMM_PLAN=1" "AMGT_DENSE_FROM_BIN=3" "AMGT_DENSE_FROM_BIN=4"; do
  echo "$v $(env $v python tools/spgemm_time.py cfg4 5 2>&1 | tail -1)" >> $O/cfg4_knobs2.txt
done
cat $O/cfg4_knobs2.txt
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -k regex:'^k_' --csv --log-file $O/cfg4_launches3.csv python tools/profile_cfg4.py 2 > $O/cfg4_ncu3.log 2>&1
python tools/ncu_sum_launches.py $O/cfg4_launches3.csv --per-launch > $O/cfg4_launches3.txt 2>&1
