timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "ld or sym or pair or tri" 2>&1 | tail -1
for w in ld32k fastid20m; do for r in 1 2; do for l in libsnp.so libsnp_head.so; do
  SNP_LIB_PATH=$PWD/paper_conf_ipps_binderlp19_b200/$l timeout 600 python bench.py --workload $w --steps 5 --no-cpu-baseline --no-e2e 2>/dev/null | python -c "
import sys, json; d = json.loads(sys.stdin.readline()); print('$w', '$l', d['ms_per_step'], d['roofline']['kernel_ms'], d['roofline']['frac'], d['clocks']['sm_mhz'], d['clocks']['reasons'])"
done; done; done
