cd $GRAFT_REPO_ROOT; O=gpurun_out/r2late; mkdir -p $O
for v in s256_8 s256_16 s512_16; do
  echo "== $v"
  AMGT_LIB_PATH=$PWD/paper_conf_sc_luzwflcy0c024_b200/libamgt_$v.so python tools/r2late/sym_var.py 2>&1 | tail -1
  AMGT_LIB_PATH=$PWD/paper_conf_sc_luzwflcy0c024_b200/libamgt_$v.so python tools/r2late/setup_time.py cfg3 3 2>&1 | tail -1 | cut -c1-220
done
AMGT_TRACE=1 python tools/r2late/sym_var.py 2>&1 | grep trace | tail -8
