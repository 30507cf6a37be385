set -x
timeout 900 python -m pytest tests -m gpu -q -x > gpurun_out/pytest_gpu4.log 2>&1; echo pytest=$?
tail -n 5 gpurun_out/pytest_gpu4.log
for w in fastid1m ld32k ld2k; do
timeout 300 python bench.py --workload $w --steps 10 --warmup 3 --variant tc --no-cpu-baseline --no-e2e > gpurun_out/bench_${w}_tc4.log 2>&1
tail -c 900 gpurun_out/bench_${w}_tc4.log
done
timeout 900 ncu --set full --clock-control none --import-source on -k regex:bitgemm_tc4 -s 4 -c 1 -o gpurun_out/prof_fastid_tc4 python bench.py --steps 2 --warmup 3 --variant tc --no-cpu-baseline --no-e2e > gpurun_out/ncu_full_tc4.log 2>&1; echo ncu=$?
timeout 900 ncu --set full --clock-control none --import-source on -k regex:bitgemm_tc4 -s 1 -c 1 -o gpurun_out/prof_ld32k_tc4 python bench.py --workload ld32k --steps 1 --warmup 3 --variant tc --no-cpu-baseline --no-e2e > gpurun_out/ncu_full_tc4_ld.log 2>&1; echo ncu=$?
