# Evidence run for profiles/: launch list of the default bench command, ncu --set full of the
# top kernels, a default bench line with cpu_baseline + e2e.  (1 GPU; never multi-rank.)
set -x
mkdir -p gpurun_out/prof
timeout 900 python bench.py > gpurun_out/prof/bench_default.json 2> gpurun_out/prof/bench_default.err; echo bench=$?
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -k "regex:pack_|popc|tc4|best_|bitgemm|fastid" -c 400 --csv --log-file gpurun_out/prof/launches_fastid1m.csv python bench.py --steps 3 --warmup 3 --no-cpu-baseline --no-e2e --no-graph > /dev/null 2>&1; echo ncu1=$?
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -k "regex:pack_|popc|tc4|best_|bitgemm|fastid" -c 200 --csv --log-file gpurun_out/prof/launches_ld32k.csv python bench.py --workload ld32k --steps 2 --warmup 3 --no-cpu-baseline --no-e2e --no-graph > /dev/null 2>&1; echo ncu2=$?
timeout 900 ncu --set full --clock-control none --import-source on -k regex:fastid_tc4 -s 4 -c 1 -o gpurun_out/prof/full_fastid1m python bench.py --steps 2 --warmup 3 --no-cpu-baseline --no-e2e --no-graph > /dev/null 2>&1; echo ncu3=$?
timeout 900 ncu --set full --clock-control none --import-source on -k regex:gemm_tc4 -s 2 -c 1 -o gpurun_out/prof/full_ld32k python bench.py --workload ld32k --steps 1 --warmup 3 --no-cpu-baseline --no-e2e --no-graph > /dev/null 2>&1; echo ncu4=$?
timeout 900 ncu --set full --clock-control none --import-source on -k regex:bitgemm_popc -s 2 -c 1 -o gpurun_out/prof/full_fastid1m_popc python bench.py --variant popc --steps 2 --warmup 3 --no-cpu-baseline --no-e2e --no-graph > /dev/null 2>&1; echo ncu5=$?
ls -la gpurun_out/prof
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -k "regex:pack_|popc|tc4|best_|bitgemm|fastid" -c 60 --csv --log-file gpurun_out/prof/launches_ld2k.csv python bench.py --workload ld2k --steps 3 --warmup 3 --no-cpu-baseline --no-e2e --no-graph > /dev/null 2>&1; echo ncu6=$?
timeout 600 ncu --set full --clock-control none --import-source on -k regex:gemm_tc4 -s 3 -c 1 -o gpurun_out/prof/full_ld2k python bench.py --workload ld2k --steps 2 --warmup 3 --no-cpu-baseline --no-e2e --no-graph > /dev/null 2>&1; echo ncu7=$?
