# LD iteration: LD parity tests, LD-32K / LD-2K benches
set -x
timeout 900 python -m pytest tests -m gpu -q -x -k "ld or LD" > gpurun_out/pytest_ld.log 2>&1; echo pytest_ld=$?; tail -n 3 gpurun_out/pytest_ld.log
timeout 300 python bench.py --workload ld32k --steps 5 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/bench_ld32k.log 2>&1
timeout 300 python bench.py --workload ld2k --steps 50 --warmup 5 --no-cpu-baseline --no-e2e > gpurun_out/bench_ld2k.log 2>&1
python scripts/summarize.py gpurun_out/bench_ld32k.log gpurun_out/bench_ld2k.log
