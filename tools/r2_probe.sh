set -x
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out/r2
nproc; free -g | head -2
( time timeout 900 python bench.py --config cfg3 --steps 20 --warmup 5 > gpurun_out/r2/probe_cfg3.json 2> gpurun_out/r2/probe_cfg3.err ) 2> gpurun_out/r2/probe_cfg3.time
( time timeout 900 python bench.py --impl reference --config cfg3 --steps 1 --warmup 0 > gpurun_out/r2/probe_ref_cfg3.json 2> gpurun_out/r2/probe_ref_cfg3.err ) 2> gpurun_out/r2/probe_ref_cfg3.time
tail -3 gpurun_out/r2/*.time
