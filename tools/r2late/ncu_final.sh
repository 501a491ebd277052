cd $GRAFT_REPO_ROOT; O=gpurun_out/r2late/ncufinal; mkdir -p $O
timeout 1200 ncu --set full --clock-control none -k regex:'k_plan_flat|k_gdense_pairs|k_sym_block|k_plan_zero' -c 6 -o /tmp/final_spgemm python tools/profile_cfg4.py 1 > $O/ncu.log 2>&1
ncu -i /tmp/final_spgemm.ncu-rep --page details --csv > $O/spgemm_cfg4_details.csv 2>&1
python tools/ncu_brief.py /tmp/final_spgemm.ncu-rep > $O/spgemm_cfg4_brief.txt 2>&1
