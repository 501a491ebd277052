# round-2 final measurement batch: GPU suite, smoke, bench x2 (the driver's command), reference
# arm, bench launch list (ncu), forced-partition config 5 at one rank, 512^3 virtual-rank overhead
cd $GRAFT_REPO_ROOT; O=gpurun_out/r2final; mkdir -p $O
timeout 1800 python -m pytest tests -q -m gpu > $O/gpu_tests.log 2>&1; echo "rc=$?" >> $O/gpu_tests.log
python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke.log 2>&1; echo "rc=$?" >> $O/smoke.log
timeout 900 python bench.py > $O/bench_1.json 2> $O/bench_1.err
timeout 900 python bench.py > $O/bench_2.json 2> $O/bench_2.err
timeout 900 python bench.py --impl reference > $O/bench_ref.json 2> $O/bench_ref.err
timeout 1500 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:"^k_" -c 20000 --csv --log-file $O/bench_launches.csv python bench.py --steps 2 --warmup 3 --no-cpu-baseline --no-cfg4 > $O/bench_ncu.log 2>&1
timeout 900 python bench.py --force-dist --config cfg5 --steps 3 --warmup 3 > $O/bench_cfg5_forced.json 2> $O/bench_cfg5_forced.err
timeout 1500 python tools/dist_overhead.py --n 512 --cycles 10 --agg-rows 262144 > $O/dist_overhead_512.jsonl 2> $O/dist_overhead_512.err
echo done > $O/done
