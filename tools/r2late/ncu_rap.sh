cd $GRAFT_REPO_ROOT; O=gpurun_out/r2late; mkdir -p $O
timeout 900 ncu --set full --import-source on --clock-control none --nvtx --nvtx-include 'setup/' -k regex:'k_numeric<|k_numeric_b1|k_csr2mbsr<1' -c 3 -o $O/rap_full python tools/setup_kernels.py cfg3 > $O/rap_full.log 2>&1
ncu -i $O/rap_full.ncu-rep --page details --csv > $O/rap_full.csv 2>&1
ncu -i $O/rap_full.ncu-rep --page raw --csv > $O/rap_raw.csv 2>&1
