timeout 1200 python -m pytest tests/test_gpu_parity.py -q -x -k "ld or sym or general or ties or search_chunked" 2>&1 | tail -1
for w in ld32k ld2k fastid20m; do st=20; [ $w = fastid20m ] && st=5
  timeout 600 python bench.py --workload $w --steps $st --no-cpu-baseline --no-e2e 2>/dev/null | python -c "
import sys, json; d = json.loads(sys.stdin.readline()); print('$w', round(d['ms_per_step'], 5), round(d['roofline']['kernel_ms'], 5), round(d['roofline']['frac'], 4), d['clocks']['reasons'])"
done
