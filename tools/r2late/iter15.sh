cd $GRAFT_REPO_ROOT; O=gpurun_out/r2late; mkdir -p $O
timeout 900 python -m pytest tests/test_gpu_convert.py -x -q -m gpu > $O/t15.log 2>&1; tail -2 $O/t15.log
python tools/r2late/setup_time.py cfg3 3 2>&1 | tail -1
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --nvtx --nvtx-include 'setup/' -k regex:'^k_csr2mbsr' --csv --log-file $O/kconv.csv python tools/setup_kernels.py cfg3 > /dev/null 2>&1
python tools/ncu_sum_launches.py $O/kconv.csv | head -5
