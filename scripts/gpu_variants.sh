# gpu_variants.sh V1 V2 ...: run the fastid experiment + search parity tests per library variant
cp paper_conf_ipps_binderlp19_b200/libsnp.so /tmp/libsnp_base.so
for v in "$@"; do
  if [ "$v" = base ]; then cp /tmp/libsnp_base.so paper_conf_ipps_binderlp19_b200/libsnp.so; else cp paper_conf_ipps_binderlp19_b200/libsnp_$v.so paper_conf_ipps_binderlp19_b200/libsnp.so; fi
  echo "== $v"
  timeout 600 python -m pytest tests -m gpu -x -q -k "search or fastid" 2>&1 | tail -1
  timeout 300 python scripts/fastid_exp.py 2>&1 | python -c "
import sys,json
for l in sys.stdin:
    if l.startswith('{'):
        d=json.loads(l); print({k:round(v['us'],1) for k,v in d.items()})
    else: print(l.rstrip())
"
done
cp /tmp/libsnp_base.so paper_conf_ipps_binderlp19_b200/libsnp.so
