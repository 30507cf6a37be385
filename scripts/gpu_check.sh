#!/bin/bash
# Quick state check on one B200: GPU tests, smoke, bench lines for every workload.
mkdir -p gpurun_out/chk
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv
timeout 1500 python -m pytest tests -m gpu -q -x > gpurun_out/chk/pytest_gpu.log 2>&1; echo pytest=$?
tail -3 gpurun_out/chk/pytest_gpu.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/chk/smoke.log 2>&1; echo smoke=$?
timeout 900 python bench.py > gpurun_out/chk/bench_default.json 2> gpurun_out/chk/bench_default.err; echo bench=$?
for w in ld2k ld32k fastid20m; do timeout 900 python bench.py --workload $w --steps 10 --no-cpu-baseline > gpurun_out/chk/bench_$w.json 2> gpurun_out/chk/bench_$w.err; echo $w=$?; done
cat gpurun_out/chk/bench_*.json | cut -c1-400
