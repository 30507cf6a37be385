# gpu_ldvariants.sh V1 V2 ...: LD parity subset + LD-32K / LD-2K timing per library variant
cp paper_conf_ipps_binderlp19_b200/libsnp.so /tmp/libsnp_base.so
for v in "$@"; do
  if [ "$v" = base ]; then cp /tmp/libsnp_base.so paper_conf_ipps_binderlp19_b200/libsnp.so; else cp paper_conf_ipps_binderlp19_b200/libsnp_$v.so paper_conf_ipps_binderlp19_b200/libsnp.so; fi
  echo "== $v"
  timeout 600 python -m pytest tests -m gpu -x -q -k "ld and not 32k" 2>&1 | tail -1
  timeout 300 python scripts/ld_exp.py 2>&1 | tail -1
  M=2048 K=4096 timeout 300 python scripts/ld_exp.py 2>&1 | tail -1
done
cp /tmp/libsnp_base.so paper_conf_ipps_binderlp19_b200/libsnp.so
