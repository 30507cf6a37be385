#!/bin/bash
# configs[4] few-query sweep at HEAD (stream vs tensor variant, best-only search) for the a7 threshold,
# plus the tensor path at the paper's profile lengths (16-128-byte rows)
mkdir -p gpurun_out/sweep
timeout 1500 python scripts/sweep.py --M 1,2,3,4,6,8,16,32,64 --N 1000000,4000000,20000000 --K 2048,4096,8192,16384 --max-popc-s 0.25 > gpurun_out/sweep/sweep_few.jsonl 2> gpurun_out/sweep/sweep_few.txt; echo sweep=$?
timeout 600 python scripts/sweep.py --M 1,4,32 --N 20000000 --K 128,256,512,1024 --tight --max-popc-s 0.25 > gpurun_out/sweep/sweep_paper.jsonl 2> gpurun_out/sweep/sweep_paper.txt; echo paper=$?
timeout 600 python scripts/sweep.py --M 32 --N 20000000 --K 128,256,512,1024 --tight --counts --max-popc-s 0.05 > gpurun_out/sweep/sweep_paper_counts.jsonl 2> gpurun_out/sweep/sweep_paper_counts.txt; echo paperc=$?
cat gpurun_out/sweep/*.txt | head -150
