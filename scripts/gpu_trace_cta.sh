timeout 600 python bench.py --steps 20 --no-cpu-baseline 2>&1 | python -c "
import sys, json; d = json.loads(sys.stdin.readline()); e=d['e2e']; print(d['ms_per_step'], e['ms_per_step'], e['value'], e.get('result_matches_device_step'), e['h2d_bytes_per_step'], e['d2h_bytes_per_step'])"
bash scripts/gpu_mg.sh 2>&1 | cut -c1-150
