for r in 1 2; do for l in libsnp.so libsnp_ns2.so libsnp_ns4.so; do
  SNP_LIB_PATH=$PWD/paper_conf_ipps_binderlp19_b200/$l timeout 600 python bench.py --workload ld32k --steps 10 --no-cpu-baseline --no-e2e 2>/dev/null | python -c "
import sys, json
try:
    d = json.loads(sys.stdin.readline()); print('ld32k', '$l', round(d['ms_per_step'], 4), round(d['roofline']['kernel_ms'], 4), d['clocks']['sm_mhz'], d['clocks']['reasons'])
except Exception as e: print('$l failed')"
done; done
