cd $GRAFT_REPO_ROOT; O=gpurun_out/r2late; mkdir -p $O
for v in 0 1; do echo "HW=$v $(AMGT_NUM_HW=$v python tools/r2late/setup_time.py cfg3 3 2>&1 | tail -1)"; done
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --nvtx --nvtx-include 'setup/' -k regex:'^k_' --csv --log-file $O/setup3.csv python tools/setup_kernels.py cfg3 > $O/setup3.log 2>&1
python tools/ncu_sum_launches.py $O/setup3.csv > $O/setup3.txt 2>&1; head -24 $O/setup3.txt
