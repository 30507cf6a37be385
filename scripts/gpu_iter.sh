# build-measure iteration: quick TC parity, full GPU tests, benches, one ncu capture
set -x
timeout 120 python scripts/tc_quick.py > gpurun_out/tc_quick.log 2>&1; echo tcq=$?; tail -n 2 gpurun_out/tc_quick.log
timeout 900 python -m pytest tests -m gpu -q -x > gpurun_out/pytest_gpu.log 2>&1; echo pytest=$?; tail -n 3 gpurun_out/pytest_gpu.log
for w in fastid1m ld32k ld2k; do
timeout 300 python bench.py --workload $w --steps 10 --warmup 3 --variant tc --no-cpu-baseline --no-e2e > gpurun_out/bench_${w}.log 2>&1
done
python scripts/summarize.py gpurun_out/bench_fastid1m.log gpurun_out/bench_ld32k.log gpurun_out/bench_ld2k.log
if [ -n "$NCU" ]; then
timeout 900 ncu --set full --clock-control none --import-source on -k regex:${KREGEX:-tc4_kernel} -s 4 -c 1 -o gpurun_out/prof_iter python bench.py --steps 2 --warmup 3 --variant tc --no-cpu-baseline --no-e2e > gpurun_out/ncu_iter.log 2>&1; echo ncu=$?
fi
