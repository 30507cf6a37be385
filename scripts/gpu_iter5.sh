set -x
timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1; echo pytest=$?; tail -n 3 gpurun_out/pytest_gpu.log
timeout 300 python scripts/ld_exp.py > gpurun_out/ldexp.log 2>&1
M=2048 K=4096 timeout 300 python scripts/ld_exp.py > gpurun_out/ldexp2k.log 2>&1
timeout 300 python scripts/fastid_exp.py > gpurun_out/fexp.log 2>&1
for f in gpurun_out/ldexp*.log gpurun_out/fexp.log; do echo $f; cat $f; done
