cd $GRAFT_REPO_ROOT; O=gpurun_out/r2late; mkdir -p $O
timeout 900 ncu --set full --import-source on --clock-control none --nvtx --nvtx-include 'setup/' -k regex:'^k_numeric$' -c 1 -o $O/rap_num python tools/setup_kernels.py cfg3 > $O/rap_num.log 2>&1
timeout 900 ncu --set full --import-source on --clock-control none --nvtx --nvtx-include 'setup/' -k regex:'^k_csr2mbsr$' --launch-skip 1 -c 1 -o $O/conv_fill python tools/setup_kernels.py cfg3 > $O/conv_fill.log 2>&1
for f in rap_num conv_fill; do ncu -i $O/$f.ncu-rep --page details --csv > $O/$f.csv 2>&1; ncu -i $O/$f.ncu-rep --page source --csv > $O/${f}_src.csv 2>&1; done
