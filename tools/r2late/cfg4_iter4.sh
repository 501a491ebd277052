cd $GRAFT_REPO_ROOT; O=gpurun_out/r2late; mkdir -p $O
timeout 900 python -m pytest tests/test_gpu_spgemm.py -x -q -m gpu > $O/t_spgemm4.log 2>&1; tail -3 $O/t_spgemm4.log
rm -f $O/cfg4_knobs4.txt
for v in "AMGT_PLAN_HINTS=0" "AMGT_PLAN_HINTS=1" "AMGT_PLAN_HINTS=2" "AMGT_PLAN_HINTS=3" "AMGT_PLAN_HINTS=3 AMGT_PLAN_BAND_MB=6" "AMGT_PLAN_HINTS=3 AMGT_PLAN_BAND_MB=1000"; do
  echo "$v $(env $v python tools/spgemm_time.py cfg4 5 2>&1 | tail -1 | cut -c1-300)" >> $O/cfg4_knobs4.txt
done
cat $O/cfg4_knobs4.txt
timeout 900 ncu --set full --clock-control none -k regex:'k_plan_flat' -c 1 -o $O/plan_flat_full python tools/profile_cfg4.py 1 > $O/ncu_pf.log 2>&1
ncu -i $O/plan_flat_full.ncu-rep --page details --csv > $O/plan_flat_full.csv 2>&1
