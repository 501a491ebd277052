cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out/r2d
timeout 900 python tools/dist_overhead.py --n 512 --cycles 2 --agg-rows 262144 --G 8 > gpurun_out/r2d/g8_a.jsonl 2> gpurun_out/r2d/g8_a.err
AMGT_CONV_STAGE=0 timeout 900 python tools/dist_overhead.py --n 512 --cycles 2 --agg-rows 262144 --G 8 > gpurun_out/r2d/g8_nostage.jsonl 2> gpurun_out/r2d/g8_nostage.err
CUDA_LAUNCH_BLOCKING=1 timeout 900 python tools/dist_overhead.py --n 512 --cycles 2 --agg-rows 262144 --G 8 > gpurun_out/r2d/g8_block.jsonl 2> gpurun_out/r2d/g8_block.err
