cd $GRAFT_REPO_ROOT; O=gpurun_out/r2late; mkdir -p $O
timeout 900 python -m pytest tests/test_gpu_spgemm.py tests/test_gpu_vcycle.py -x -q -m gpu > $O/t13.log 2>&1; tail -2 $O/t13.log
for v in 0 1; do echo "PIPE=$v $(AMGT_B1_PIPE=$v python tools/r2late/setup_time.py cfg3 3 2>&1 | tail -1)"; done
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --nvtx --nvtx-include 'setup/' -k regex:'^k_numeric_b1' --csv --log-file $O/kb1.csv python tools/setup_kernels.py cfg3 > /dev/null 2>&1
python tools/ncu_sum_launches.py $O/kb1.csv | head -5
