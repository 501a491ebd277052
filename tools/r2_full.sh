# full GPU suite + smoke + ncu traffic captures (cfg3 level-1 SpMV, cfg4 SpGEMM) + forced-partition bench
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out/r2
python __graft_entry__.py build > gpurun_out/r2/build.log 2>&1
timeout 1500 python -m pytest tests -q -m gpu > gpurun_out/r2/gpu_tests.log 2>&1; echo "rc=$?" >> gpurun_out/r2/gpu_tests.log
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r2/smoke.log 2>&1; echo "rc=$?" >> gpurun_out/r2/smoke.log
timeout 900 ncu --set full --clock-control none -k regex:'k_spmv_rows<double' -c 4 -f -o gpurun_out/r2/ncu_spmv_cfg3 python tools/ncu_traffic.py run cfg3 > gpurun_out/r2/ncu_cfg3.log 2>&1
timeout 900 ncu --set full --clock-control none --nvtx --nvtx-include 'amgt_spgemm/' -f -o gpurun_out/r2/ncu_spgemm_cfg4 python tools/ncu_traffic.py run cfg4 > gpurun_out/r2/ncu_cfg4.log 2>&1
timeout 900 python bench.py --force-dist --config cfg5 --steps 3 --warmup 3 --cycles 10 > gpurun_out/r2/bench_dist_cfg5.json 2> gpurun_out/r2/bench_dist_cfg5.err; echo "rc=$?" >> gpurun_out/r2/bench_dist_cfg5.err
