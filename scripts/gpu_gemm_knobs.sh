#!/bin/bash
# gemm_tc4 compile-time knobs re-measured after the per-stage MMA issue and write-back stores
for w in ld32k ld2k fastid20m; do for l in libsnp.so libsnp_gh2.so libsnp_np8.so libsnp_x2e.so; do
  st=10; [ $w = fastid20m ] && st=4
  SNP_LIB_PATH=$PWD/paper_conf_ipps_binderlp19_b200/$l timeout 600 python bench.py --workload $w --steps $st --no-cpu-baseline --no-e2e 2>/dev/null | python -c "
import sys, json
try:
    d = json.loads(sys.stdin.readline()); print('$w', '$l', round(d['ms_per_step'], 5), round(d['roofline']['kernel_ms'], 5), round(d['roofline']['frac'], 4), d['clocks']['reasons'])
except Exception as e: print('$w', '$l', 'failed', e)"
done; done
