set -x
timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1; echo pytest=$?; tail -n 3 gpurun_out/pytest_gpu.log
timeout 300 python scripts/fastid_exp.py > gpurun_out/fexp.log 2>&1
timeout 300 python bench.py --steps 100 --no-cpu-baseline > gpurun_out/bench_f.json 2>gpurun_out/bench_f.err
python - <<'PY'
import json
for l in open("gpurun_out/fexp.log"):
    if l.startswith("{"): print({k: round(v["us"], 1) for k, v in json.loads(l).items()})
b = json.loads(open("gpurun_out/bench_f.json").read().strip().splitlines()[-1])
print("bench", b["ms_per_step"], b["value"], b["roofline"]["frac"], b["roofline"]["kernel_ms"], b["e2e"]["ms_per_step"])
PY
