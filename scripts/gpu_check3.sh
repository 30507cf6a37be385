set -x
timeout 120 python scripts/tc_quick.py > gpurun_out/tc_quick_f4.log 2>&1; echo tcq=$?
cat gpurun_out/tc_quick_f4.log
SNP_TC_KIND=i8 timeout 120 python scripts/tc_quick.py > gpurun_out/tc_quick_i8.log 2>&1; echo tcq8=$?
tail -n 3 gpurun_out/tc_quick_i8.log
timeout 900 python -m pytest tests -m gpu -q -x > gpurun_out/pytest_gpu3.log 2>&1; echo pytest=$?
tail -n 30 gpurun_out/pytest_gpu3.log
for w in fastid1m ld32k; do
timeout 300 python bench.py --workload $w --steps 10 --warmup 3 --variant tc --no-cpu-baseline --no-e2e > gpurun_out/bench_${w}_tc4.log 2>&1
tail -c 1500 gpurun_out/bench_${w}_tc4.log
done
