mkdir -p gpurun_out/prof
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -k "regex:pack_|popc|tc4|best_|bitgemm|fastid" -c 60 --csv --log-file gpurun_out/prof/launches_ld2k.csv python bench.py --workload ld2k --steps 3 --warmup 3 --no-cpu-baseline --no-e2e --no-graph > /dev/null 2>&1; echo ncu1=$?
timeout 600 ncu --set full --clock-control none --import-source on -k regex:gemm_tc4 -s 3 -c 1 -o gpurun_out/prof/full_ld2k python bench.py --workload ld2k --steps 2 --warmup 3 --no-cpu-baseline --no-e2e --no-graph > /dev/null 2>&1; echo ncu2=$?
SNP_TRACE=1 M=2048 NB=4096 timeout 300 python scripts/trace_gemm.py 2>&1 | tail -30
