cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out/r2w
for pat in 53 62 71 44; do
AMGT_W2_PAT=$pat timeout 600 python tools/sweep_cfg.py cfg3 3 "w2:4:-1" > gpurun_out/r2w/w2_cfg3_$pat.jsonl 2> gpurun_out/r2w/w2_cfg3_$pat.err
done
AMGT_W2_PAT=53 timeout 600 python tools/sweep_cfg.py cfg2 5 "w2:4:-1,w2:2:-1" > gpurun_out/r2w/w2_cfg2.jsonl 2> gpurun_out/r2w/w2_cfg2.err
echo done > gpurun_out/r2w/done
