# round-2 measurement batch: full GPU suite, smoke, bench lines (driver command), reference arm,
# bench launch list, distributed overhead, forced-partition cfg5 point
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out/r2m
python __graft_entry__.py build > gpurun_out/r2m/build.log 2>&1
timeout 1500 python -m pytest tests -q -m gpu > gpurun_out/r2m/gpu_tests.log 2>&1; echo "rc=$?" >> gpurun_out/r2m/gpu_tests.log
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r2m/smoke.log 2>&1; echo "rc=$?" >> gpurun_out/r2m/smoke.log
for i in 1 2; do
  ( time timeout 1200 python bench.py --gpus 1 --steps 20 --warmup 5 > gpurun_out/r2m/bench_$i.json 2> gpurun_out/r2m/bench_$i.err ) 2> gpurun_out/r2m/bench_$i.time
done
( time timeout 1200 python bench.py --impl reference --gpus 1 --steps 20 --warmup 5 > gpurun_out/r2m/bench_ref.json 2> gpurun_out/r2m/bench_ref.err ) 2> gpurun_out/r2m/bench_ref.time
timeout 1500 ncu --metrics gpu__time_duration.sum --clock-control none -c 20000 --csv --log-file gpurun_out/r2m/bench_launches.csv python bench.py --steps 2 --warmup 3 --no-cpu-baseline --no-cfg4 > gpurun_out/r2m/bench_ncu.log 2>&1
timeout 1500 python tools/dist_overhead.py --n 512 --cycles 10 --agg-rows 262144 > gpurun_out/r2m/dist_overhead_512.jsonl 2> gpurun_out/r2m/dist_overhead_512.err
timeout 1200 python bench.py --force-dist --config cfg5 --steps 5 --warmup 3 > gpurun_out/r2m/bench_cfg5_forced.json 2> gpurun_out/r2m/bench_cfg5_forced.err
