#!/bin/bash
# per-stage elected MMA issue (libsnp.so) vs HEAD before it (libsnp_head.so): GPU tests, FastID shapes, LD bench lines
timeout 1500 python -m pytest tests -m gpu -q -x 2>&1 | tail -2
for cfg in "NQ=64 ND=1000000 K=4096 COUNTS=1 NOPS=2" "NQ=8 ND=20000000 K=4096 COUNTS=0 NOPS=1" "NQ=32 ND=20000000 K=2048 COUNTS=0 NOPS=1" "TIGHT=1 NQ=32 ND=20000000 K=128 COUNTS=0 NOPS=1"; do
  echo "== $cfg"
  for r in 1 2; do for l in libsnp.so libsnp_head.so; do
    env $cfg SNP_LIB_PATH=$PWD/paper_conf_ipps_binderlp19_b200/$l timeout 120 python scripts/ab_fastid.py 2>&1 | python -c "
import sys, json
for l in sys.stdin:
    try: d = json.loads(l)
    except Exception: print(l.strip()[:200]); continue
    print(d.get('lib'), d.get('us_best'), d.get('hbm_frac'))"
  done; done
done
for w in ld2k ld32k; do for l in libsnp.so libsnp_head.so; do
  SNP_LIB_PATH=$PWD/paper_conf_ipps_binderlp19_b200/$l timeout 600 python bench.py --workload $w --steps 10 --no-cpu-baseline --no-e2e 2>/dev/null | python -c "
import sys, json; d = json.loads(sys.stdin.readline()); print('$w', '$l', d['ms_per_step'], d['roofline']['kernel_ms'], d['roofline']['frac'])"
done; done
M=2048 timeout 300 python scripts/ld_parts.py
