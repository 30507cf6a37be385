set -x
timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1; echo pytest=$?; tail -n 15 gpurun_out/pytest_gpu.log
timeout 300 python scripts/ld_exp.py > gpurun_out/ldexp.log 2>&1; echo $?
M=2048 K=4096 timeout 300 python scripts/ld_exp.py > gpurun_out/ldexp2k.log 2>&1; echo $?
cat gpurun_out/ldexp*.log
