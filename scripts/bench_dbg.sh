for i in 1 2 3; do timeout 300 python bench.py --workload ld32k --steps 3 --no-cpu-baseline --no-e2e 2>&1 | grep -v CUDAEvent | python scripts/summarize.py /dev/stdin 2>&1 | cut -c1-150; done
for i in 1 2; do WDMODE=0 timeout 200 python scripts/ld_repro7.py 2>&1 | tail -1; done
timeout 300 python bench.py --workload ld2k --steps 3 --no-cpu-baseline --no-e2e 2>&1 | grep -v CUDAEvent | python scripts/summarize.py /dev/stdin 2>&1 | cut -c1-150
