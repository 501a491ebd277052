# ncu --set full of the config-3 setup's conversion (A_1 count + fill), R*(AP) numeric and the first symbolic pass
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out/r2f
timeout 900 ncu --set full --import-source on --clock-control none --nvtx --nvtx-include 'setup/' -k regex:k_csr2mbsr -c 2 -o gpurun_out/r2f/conv python tools/setup_kernels.py cfg3 > gpurun_out/r2f/conv.log 2>&1
timeout 900 ncu --set full --import-source on --clock-control none --nvtx --nvtx-include 'setup/' -k regex:'k_numeric<|k_sym_flat' -c 2 -o gpurun_out/r2f/rap python tools/setup_kernels.py cfg3 > gpurun_out/r2f/rap.log 2>&1
echo done > gpurun_out/r2f/done
