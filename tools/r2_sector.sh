# sector-skipping FP64 SpMV vs the full-tile loads, x L2 fetch granularity; + ncu DRAM bytes
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out/r2s
for c in cfg3 cfg2; do
  for v in 0 4; do
    for f in "" 32 64; do
      AMGT_SPMV_VARIANT=$v AMGT_L2_FETCH=$f timeout 300 python tools/sector_probe.py $c 10 >> gpurun_out/r2s/probe.jsonl 2>> gpurun_out/r2s/probe.err
    done
  done
done
M=gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum
for v in 0 4; do for f in "" 32; do
AMGT_SPMV_VARIANT=$v AMGT_L2_FETCH=$f timeout 600 ncu --metrics $M --clock-control none -k regex:k_spmv_rows --csv --log-file gpurun_out/r2s/ncu_v${v}_f${f}.csv python tools/sector_probe.py cfg3 2 > /dev/null 2>&1
done; done
echo done > gpurun_out/r2s/done
