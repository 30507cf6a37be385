set -x
timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1; echo pytest=$?; tail -n 5 gpurun_out/pytest_gpu.log
timeout 300 python scripts/fastid_exp.py > gpurun_out/fexp.log 2>&1
timeout 300 python bench.py --steps 100 --no-cpu-baseline > gpurun_out/bench_f.json 2>gpurun_out/bench_f.err
cat gpurun_out/fexp.log; cut -c1-400 gpurun_out/bench_f.json; tail -3 gpurun_out/bench_f.err
