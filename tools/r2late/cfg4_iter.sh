# SpGEMM tests, then cfg4 timings under knob variants, then a launch list of the default
cd $GRAFT_REPO_ROOT; O=gpurun_out/r2late; mkdir -p $O
timeout 900 python -m pytest tests/test_gpu_spgemm.py tests/test_gpu_bitmap_exhaustive.py -x -q -m gpu > $O/t_spgemm.log 2>&1; tail -3 $O/t_spgemm.log
for v in "AMGT_GDENSE=0" "AMGT_GDENSE=1" "AMGT_DENSE_FROM_BIN=3" "AMGT_DENSE_FROM_BIN=4" "AMGT_DENSE_FROM_BIN=6"; do
  echo "$v $(env $v python tools/spgemm_time.py cfg4 5 2>&1 | head -1)" >> $O/cfg4_knobs.txt
done
cat $O/cfg4_knobs.txt
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -k regex:'^k_' --csv --log-file $O/cfg4_launches2.csv python tools/profile_cfg4.py 2 > $O/cfg4_ncu2.log 2>&1
python tools/ncu_sum_launches.py $O/cfg4_launches2.csv --per-launch > $O/cfg4_launches2.txt 2>&1
