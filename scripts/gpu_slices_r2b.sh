#!/bin/bash
# > 64 queries: 64-query slices of the FastID kernel vs the general kernel (SNP_SEARCH_SLICES=0), and
# <= 16 queries on long profiles: K-chunked FastID passes vs the general kernel (SNP_SEARCH_KCHUNK=0), at HEAD
mkdir -p gpurun_out/sweep
timeout 900 python scripts/sweep.py --M 128,256,1024 --N 4000000 --K 2048,4096,8192 --max-popc-s 0.01 > /dev/null 2> gpurun_out/sweep/slices_on.txt
SNP_SEARCH_SLICES=0 timeout 900 python scripts/sweep.py --M 128,256,1024 --N 4000000 --K 2048,4096,8192 --max-popc-s 0.01 > /dev/null 2> gpurun_out/sweep/slices_off.txt
timeout 900 python scripts/sweep.py --M 4,8,16,32 --N 4000000 --K 16384 --max-popc-s 0.01 > /dev/null 2> gpurun_out/sweep/kchunk_on.txt
SNP_SEARCH_KCHUNK=0 timeout 900 python scripts/sweep.py --M 4,8,16,32 --N 4000000 --K 16384 --max-popc-s 0.01 > /dev/null 2> gpurun_out/sweep/kchunk_off.txt
paste gpurun_out/sweep/slices_on.txt gpurun_out/sweep/slices_off.txt | cut -f1-4,11 ; paste gpurun_out/sweep/kchunk_on.txt gpurun_out/sweep/kchunk_off.txt | cut -f1-4,11
