mkdir -p gpurun_out/prof
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -k "regex:gemm|best_|row_popc|fastid" -c 40 --csv --log-file gpurun_out/prof/launches_fastid20m.csv python bench.py --workload fastid20m --steps 1 --warmup 3 --no-cpu-baseline --no-e2e --no-graph > /dev/null 2>&1; echo ncu=$?
