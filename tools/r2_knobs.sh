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
