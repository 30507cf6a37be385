for cfg in "TIGHT=1 NQ=32 K=1024 COUNTS=0 NOPS=1" "TIGHT=1 NQ=32 K=512 COUNTS=0 NOPS=1" "NQ=8 K=4096 COUNTS=0 NOPS=1" "NQ=32 K=2048 COUNTS=0 NOPS=1" "NQ=16 K=2048 COUNTS=1 NOPS=1"; do
  echo "== $cfg"
  for l in libsnp.so libsnp_ia.so libsnp_ns3.so libsnp_ians3.so; do
    env $cfg ND=20000000 CHECK=1 SNP_LIB_PATH=$PWD/paper_conf_ipps_binderlp19_b200/$l timeout 120 python scripts/ab_fastid.py 2>&1 | python -c "
import sys, json
for l in sys.stdin:
    try: d = json.loads(l)
    except Exception: print(l.strip()); continue
    print(d.get('lib'), d.get('us_best', ''), d.get('hbm_frac', ''), d.get('check_vs_popc', ''))"
  done
done
