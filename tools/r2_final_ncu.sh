# bench launch list (our kernels only), the driver's command shape at 2 timed steps
cd $GRAFT_REPO_ROOT; O=gpurun_out/r2final; mkdir -p $O
timeout 1500 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:'^k_' -c 20000 --csv --log-file $O/bench_launches.csv python bench.py --steps 2 --warmup 3 --no-cpu-baseline --no-cfg4 > $O/bench_ncu.log 2>&1
echo done > $O/done2
