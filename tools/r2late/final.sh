# late-round measurement batch: GPU suite, smoke, bench x2 (the driver's command), reference arm,
# bench launch list (ncu), config-4 SpGEMM traffic capture (ncu --set full), sanitizer on SpGEMM
cd $GRAFT_REPO_ROOT; O=gpurun_out/r2late/final3; mkdir -p $O
timeout 1800 python -m pytest tests -q -m gpu > $O/gpu_tests.log 2>&1; echo "rc=$?" >> $O/gpu_tests.log; tail -2 $O/gpu_tests.log
python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke.log 2>&1; echo "rc=$?" >> $O/smoke.log; tail -2 $O/smoke.log
timeout 900 python bench.py > $O/bench_1.json 2> $O/bench_1.err
timeout 900 python bench.py > $O/bench_2.json 2> $O/bench_2.err
timeout 900 python bench.py --impl reference > $O/bench_ref.json 2> $O/bench_ref.err
timeout 1500 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:"^k_" -c 20000 --csv --log-file $O/bench_launches.csv python bench.py --steps 2 --warmup 3 --no-cpu-baseline --no-cfg4 > $O/bench_ncu.log 2>&1
timeout 1500 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum --clock-control none --nvtx --nvtx-include 'amgt_spgemm/' -o /tmp/ncu_spgemm_cfg4 python tools/ncu_traffic.py run cfg4 > $O/ncu_cfg4.log 2>&1
python tools/ncu_traffic.py summarize cfg4 /tmp/ncu_spgemm_cfg4.ncu-rep > $O/ncu_cfg4_sum.log 2>&1
cp profiles/ncu_traffic_cfg4.json $O/ncu_traffic_cfg4.json
gzip -f $O/bench_launches.csv
echo done > $O/done
