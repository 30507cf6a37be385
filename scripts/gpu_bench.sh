set -x
for v in tc popc; do
  timeout 300 python bench.py --steps 50 --warmup 5 --variant $v --no-cpu-baseline > gpurun_out/bench_fastid_$v.log 2>&1; echo $v=$?
done
timeout 300 python bench.py --workload ld2k --steps 20 --variant tc --no-cpu-baseline > gpurun_out/bench_ld2k_tc.log 2>&1
timeout 600 python bench.py --workload ld32k --steps 3 --variant tc --no-cpu-baseline > gpurun_out/bench_ld32k_tc.log 2>&1
timeout 600 python bench.py --workload ld32k --steps 2 --variant popc --no-cpu-baseline --no-e2e > gpurun_out/bench_ld32k_popc.log 2>&1
cat gpurun_out/bench_*.log | cut -c1-1500
# launch list + full profile of the tc kernel on fastid
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 200 --csv --log-file gpurun_out/launches_fastid_tc.csv python bench.py --steps 2 --warmup 3 --variant tc --no-cpu-baseline --no-e2e > /dev/null 2>&1; echo ncu1=$?
timeout 900 ncu --set full --clock-control none --import-source on -k regex:bitgemm_tc -s 4 -c 1 -o gpurun_out/prof_fastid_tc python bench.py --steps 2 --warmup 3 --variant tc --no-cpu-baseline --no-e2e > gpurun_out/ncu_full.log 2>&1; echo ncu2=$?
timeout 900 ncu --set full --clock-control none --import-source on -k regex:bitgemm_popc -s 4 -c 1 -o gpurun_out/prof_fastid_popc python bench.py --steps 2 --warmup 3 --variant popc --no-cpu-baseline --no-e2e > gpurun_out/ncu_full_popc.log 2>&1; echo ncu3=$?
ls -la gpurun_out
