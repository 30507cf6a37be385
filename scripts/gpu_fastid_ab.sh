#!/bin/bash
# A/B of the FastID kernel: traces + the default bench line + skinny best-only sweep points
bash scripts/build_variant.sh tr2 "-DFASTID_TRACE2"
export SNP_LIB_PATH=$PWD/paper_conf_ipps_binderlp19_b200/libsnp_tr2.so
MODE=bestonly NQ=1 python scripts/trace_fastid2.py > gpurun_out/trace_ia_best1.txt 2>&1

unset SNP_LIB_PATH
python bench.py --steps 30 --warmup 5 --no-cpu-baseline > gpurun_out/bench_ia.json 2>gpurun_out/bench_ia.err
python scripts/sweep.py --M 1,8,32,64 --N 1000000,20000000 --K 2048,4096,8192 --max-popc-s 0 > gpurun_out/sweep_ia.jsonl 2> gpurun_out/sweep_ia.txt
