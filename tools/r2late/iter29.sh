cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out/r2late
python tools/r2late/sym_var.py 2>&1 | tail -2
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:'k_gdense_pairs|k_sym_block' --csv --log-file gpurun_out/r2late/l29.csv python tools/profile_cfg4.py 2 > /dev/null 2>&1
python tools/ncu_sum_launches.py gpurun_out/r2late/l29.csv | head -8
