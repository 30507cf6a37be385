#!/bin/bash
# Round-2 evidence pass at HEAD (1 GPU): GPU tests, smoke, bench lines (all workloads + the
# reference arm), ncu launch lists and --set full captures of the dominant kernels.
set -x
mkdir -p gpurun_out/prof
bash scripts/gpu_mg.sh > gpurun_out/prof/multirank_gloo_1gpu.txt 2>&1; echo mg=$?
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv
timeout 1500 python -m pytest tests -m gpu -q > gpurun_out/prof/pytest_gpu.log 2>&1; echo pytest=$?
tail -3 gpurun_out/prof/pytest_gpu.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/prof/smoke.log 2>&1; echo smoke=$?
timeout 900 python bench.py --steps 20 --warmup 5 > gpurun_out/prof/bench_default.json 2> gpurun_out/prof/bench_default.err; echo bench=$?
timeout 900 python bench.py --impl reference --steps 2 --warmup 1 > gpurun_out/prof/bench_reference.json 2> gpurun_out/prof/bench_reference.err
for w in ld2k ld32k fastid20m; do timeout 900 python bench.py --workload $w --steps 10 --warmup 3 --no-cpu-baseline > gpurun_out/prof/bench_$w.json 2> gpurun_out/prof/bench_$w.err; echo $w=$?; done
K="regex:pack_|popc|tc4|best_|bitgemm|fastid|stream|sym_"
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -k "$K" -c 400 --csv --log-file gpurun_out/prof/launches_fastid1m.csv python bench.py --steps 3 --warmup 3 --no-cpu-baseline --no-e2e --no-graph > /dev/null 2>&1; echo ncu1=$?
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -k "$K" -c 200 --csv --log-file gpurun_out/prof/launches_ld32k.csv python bench.py --workload ld32k --steps 2 --warmup 3 --no-cpu-baseline --no-e2e --no-graph > /dev/null 2>&1; echo ncu2=$?
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -k "$K" -c 60 --csv --log-file gpurun_out/prof/launches_ld2k.csv python bench.py --workload ld2k --steps 3 --warmup 3 --no-cpu-baseline --no-e2e --no-graph > /dev/null 2>&1; echo ncu3=$?
timeout 900 ncu --set full --clock-control none --import-source on -k regex:fastid_tc4 -s 4 -c 1 -o gpurun_out/prof/full_fastid1m python bench.py --steps 2 --warmup 3 --no-cpu-baseline --no-e2e --no-graph > /dev/null 2>&1; echo ncu4=$?
timeout 900 ncu --set full --clock-control none --import-source on -k regex:gemm_tc4 -s 2 -c 1 -o gpurun_out/prof/full_ld32k python bench.py --workload ld32k --steps 1 --warmup 3 --no-cpu-baseline --no-e2e --no-graph > /dev/null 2>&1; echo ncu5=$?
timeout 600 ncu --set full --clock-control none --import-source on -k regex:gemm_tc4 -s 3 -c 1 -o gpurun_out/prof/full_ld2k python bench.py --workload ld2k --steps 2 --warmup 3 --no-cpu-baseline --no-e2e --no-graph > /dev/null 2>&1; echo ncu6=$?
ls -la gpurun_out/prof
