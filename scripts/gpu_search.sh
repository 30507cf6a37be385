# f1 iteration: search parity tests, then fused vs separate FastID step benches
set -x
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv
timeout 900 python -m pytest tests -m gpu -q -x -k "search" > gpurun_out/pytest_search.log 2>&1; echo pytest_search=$?; tail -n 15 gpurun_out/pytest_search.log
for m in fused separate; do
timeout 300 python bench.py --steps 100 --warmup 5 --fastid-step $m --no-cpu-baseline > gpurun_out/bench_fastid_$m.log 2>&1; echo $m=$?
done
SNP_DEBUG_NOSTORE=1 timeout 300 python bench.py --steps 100 --warmup 5 --no-cpu-baseline --no-e2e > gpurun_out/bench_fastid_nostore.log 2>&1
cat gpurun_out/bench_fastid_*.log | cut -c1-2500
timeout 900 python -m pytest tests -m gpu -q -x > gpurun_out/pytest_gpu.log 2>&1; echo pytest=$?; tail -n 5 gpurun_out/pytest_gpu.log
