cd $GRAFT_REPO_ROOT; O=gpurun_out/r2late; mkdir -p $O
timeout 1200 ncu --set full --import-source on --clock-control none -k regex:'k_sym_block|k_numeric_mid|k_sym_flat|k_gdense_pairs|k_sym_warp|k_numeric_staged|k_numeric<' -c 16 -o $O/sym_full python tools/profile_cfg4.py 1 > $O/ncu_sym.log 2>&1
ncu -i $O/sym_full.ncu-rep --page details --csv > $O/sym_full.csv 2>&1
