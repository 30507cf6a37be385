mkdir -p gpurun_out/t4
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "search or fastid or stream or best" 2>&1 | tail -3
bash scripts/gpu_ab.sh selfclean libsnp.so libsnp_old.so
timeout 600 python bench.py --steps 20 --no-cpu-baseline > gpurun_out/t4/bench.json 2>/dev/null; python -c "
import json; d=json.loads(open('gpurun_out/t4/bench.json').readline()); print(d['ms_per_step'], d['roofline']['kernel_ms'], d['roofline']['frac'], d['clocks'], d['e2e']['ms_per_step'], d['gpu_launches'])"
