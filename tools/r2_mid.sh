# mid-session validation: GPU suite, smoke, bench, V-cycle launch list (cfg3, 2 cycles), level-2 SpMV ncu
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out/r2m
timeout 1800 python -m pytest tests -q -m gpu > gpurun_out/r2m/gpu_tests.log 2>&1; echo "rc=$?" >> gpurun_out/r2m/gpu_tests.log
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r2m/smoke.log 2>&1; echo "rc=$?" >> gpurun_out/r2m/smoke.log
timeout 600 python bench.py > gpurun_out/r2m/bench.json 2> gpurun_out/r2m/bench.err
M=gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum
timeout 900 ncu --metrics $M --clock-control none --csv --log-file gpurun_out/r2m/vcycle_cfg3.csv python tools/profile_vcycle.py 2 cfg3 > gpurun_out/r2m/vcycle.log 2>&1
timeout 900 ncu --set full --import-source on --clock-control none --kernel-name-base demangled -k regex:'k_spmv_rows<float' -c 3 -o gpurun_out/r2m/l2spmv python tools/profile_vcycle.py 1 cfg3 > gpurun_out/r2m/l2spmv.log 2>&1
echo done > gpurun_out/r2m/done
