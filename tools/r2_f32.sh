cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out/r2g
M=gpu__time_duration.sum,dram__bytes_read.sum
for v in 0 1 2 3; do
AMGT_SPMV_F32=$v timeout 600 ncu --metrics $M --clock-control none --kernel-name-base demangled -k regex:'k_spmv_rows<float' --csv --log-file gpurun_out/r2g/f32_$v.csv python tools/profile_vcycle.py 2 cfg3 > /dev/null 2>&1
done
for v in 0 1; do AMGT_SPMV_F32=$v timeout 300 python bench.py --steps 5 --warmup 3 --no-cpu-baseline --no-cfg4 > gpurun_out/r2g/bench_$v.json 2>/dev/null; done
echo done > gpurun_out/r2g/done
