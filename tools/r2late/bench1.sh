cd $GRAFT_REPO_ROOT; O=gpurun_out/r2late; mkdir -p $O
timeout 900 python bench.py > $O/bench_1.json 2> $O/bench_1.err; tail -2 $O/bench_1.err
python -c "import json; d=json.load(open('$O/bench_1.json')); c=d['components']; print(d['ms_per_step'], d['value'], c['setup_ms'], c['per_class_ms'], c['spgemm_roofline'], c['spgemm_cfg4']['ms'], c['spgemm_cfg4']['roofline']['frac'])"
