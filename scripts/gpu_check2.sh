set -x
timeout 120 python scripts/tc_quick.py > gpurun_out/tc_quick.log 2>&1; echo tcq=$?
cat gpurun_out/tc_quick.log
timeout 900 python -m pytest tests -m gpu -q -x > gpurun_out/pytest_gpu2.log 2>&1; echo pytest=$?
tail -n 30 gpurun_out/pytest_gpu2.log
