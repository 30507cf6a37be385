set -x
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo smoke=$?
timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1; echo pytest=$?
timeout 300 python bench.py --steps 20 --warmup 3 --cpu-seconds 5 > gpurun_out/bench1.log 2>&1; echo bench=$?
timeout 300 python bench.py --workload ld2k --steps 10 --warmup 3 --no-cpu-baseline > gpurun_out/bench_ld2k.log 2>&1; echo bench2=$?
tail -3 gpurun_out/pytest_gpu.log gpurun_out/bench1.log gpurun_out/bench_ld2k.log gpurun_out/smoke.log
