mkdir -p gpurun_out/prof
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -k "regex:pack_|popc|tc4|best_|bitgemm" -c 400 --csv --log-file gpurun_out/prof/launches_fastid1m.csv python bench.py --steps 3 --warmup 3 --no-cpu-baseline --no-e2e --no-graph > /dev/null 2>&1; echo ncu1=$?
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -k "regex:pack_|popc|tc4|best_|bitgemm" -c 200 --csv --log-file gpurun_out/prof/launches_ld32k.csv python bench.py --workload ld32k --steps 2 --warmup 3 --no-cpu-baseline --no-e2e --no-graph > /dev/null 2>&1; echo ncu2=$?
