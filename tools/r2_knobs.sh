# config-3 step under the V-cycle / SpMV measurement knobs (5 timed steps each, no CPU baseline)
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out/r2k
run() { name=$1; shift; env "$@" timeout 600 python bench.py --steps 5 --warmup 3 --no-cpu-baseline --no-cfg4 > gpurun_out/r2k/$name.json 2> gpurun_out/r2k/$name.err; }
run base
run coop AMGT_COARSE=coop
run direct AMGT_COARSE=direct
run tail512 AMGT_TAIL_BLOCKROWS=512
run var1 AMGT_SPMV_VARIANT=1
run var2 AMGT_SPMV_VARIANT=2
run var3 AMGT_SPMV_VARIANT=3
run nopdl AMGT_PDL=0
run persist0 AMGT_SPMV_PERSIST=0
run persist2 AMGT_SPMV_PERSIST=2
timeout 1500 python tools/dist_overhead.py --n 512 --cycles 10 --agg-rows 262144 > gpurun_out/r2k/dist_overhead_512.jsonl 2> gpurun_out/r2k/dist_overhead_512.err
for i in $(seq 1 12); do timeout 300 python bench.py --force-dist --config cfg2 --steps 10 --warmup 3 --no-cfg4 > gpurun_out/r2k/forced_cfg2_$i.json 2> gpurun_out/r2k/forced_cfg2_$i.err; done
