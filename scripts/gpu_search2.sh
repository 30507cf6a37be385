# quick f1 perf iteration: build in-tree, fused vs separate step, nostore, and parity of search
set -x
python -c "from paper_conf_ipps_binderlp19_b200.build import build_library; build_library()" > gpurun_out/build.log 2>&1 || tail -20 gpurun_out/build.log
timeout 600 python -m pytest tests -m gpu -q -x -k "search or fastid_all_ops or cross_variant and fastid" > gpurun_out/pytest_search.log 2>&1; echo pytest_search=$?; tail -n 5 gpurun_out/pytest_search.log
for m in fused separate; do
timeout 300 python bench.py --steps 100 --warmup 5 --fastid-step $m --no-cpu-baseline --no-e2e > gpurun_out/bench_fastid_$m.log 2>&1; echo $m=$?
done
SNP_DEBUG_NOSTORE=1 timeout 300 python bench.py --steps 100 --warmup 5 --no-cpu-baseline --no-e2e > gpurun_out/bench_fastid_nostore.log 2>&1
SNP_DEBUG_NOSTORE=1 timeout 300 python bench.py --steps 100 --warmup 5 --no-cpu-baseline --no-e2e --fastid-step separate > gpurun_out/bench_fastid_nostore_sep.log 2>&1
python scripts/summarize.py gpurun_out/bench_fastid_*.log
