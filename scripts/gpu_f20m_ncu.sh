mkdir -p gpurun_out/prof
timeout 900 ncu --set full --clock-control none --import-source on -k regex:gemm_tc4 -c 1 -o gpurun_out/prof/full_fastid20m python bench.py --workload fastid20m --steps 1 --warmup 3 --no-cpu-baseline --no-e2e --no-graph > gpurun_out/ncu_f20m.log 2>&1; echo ncu=$?
