# LD A/B per library variant: LD parity subset + LD-32K (f3 and full tiles) + LD-2K
cp paper_conf_ipps_binderlp19_b200/libsnp.so /tmp/libsnp_base.so
for v in "$@"; do
  if [ "$v" = base ]; then cp /tmp/libsnp_base.so paper_conf_ipps_binderlp19_b200/libsnp.so; else cp paper_conf_ipps_binderlp19_b200/libsnp_$v.so paper_conf_ipps_binderlp19_b200/libsnp.so; fi
  echo "== $v"
  timeout 600 python -m pytest tests -m gpu -x -q -k "ld or LD or selfld or fuzz" 2>&1 | tail -1
  timeout 300 python scripts/ld_exp.py 2>&1 | tail -1
  SNP_GEMM_SYM=0 timeout 300 python scripts/ld_exp.py 2>&1 | tail -1
  M=2048 K=4096 timeout 300 python scripts/ld_exp.py 2>&1 | tail -1
done
cp /tmp/libsnp_base.so paper_conf_ipps_binderlp19_b200/libsnp.so
