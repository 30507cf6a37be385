# Full evidence pass: GPU tests, smoke, bench lines, launch lists + ncu --set full of the top kernels.
set -x
mkdir -p gpurun_out/prof
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv
timeout 1200 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1; echo pytest=$?
tail -5 gpurun_out/pytest_gpu.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo smoke=$?
bash scripts/gpu_profiles.sh
for w in ld2k ld32k fastid20m; do timeout 600 python bench.py --workload $w --steps 10 --no-cpu-baseline > gpurun_out/prof/bench_$w.json 2> gpurun_out/prof/bench_$w.err; echo $w=$?; done
cat gpurun_out/prof/*.json | cut -c1-3000
