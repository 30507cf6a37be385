#!/bin/bash
# FastID stage-size A/B over the a7 shapes: best-only and counts+best, 512 vs 1024-bit stages
for kb in 512 1024; do
  export SNP_FASTID_KBITS=$kb
  SNP_FASTID_STREAM=0 python scripts/sweep.py --M 4,8,16,32,64 --N 1000000,20000000 --K 2048,4096,8192 --max-popc-s 0 > gpurun_out/kbm_${kb}.jsonl 2> gpurun_out/kbm_${kb}.txt
  SNP_FASTID_STREAM=0 python scripts/sweep.py --M 8,32,64 --N 1000000 --K 2048,4096,8192 --counts --max-popc-s 0 > gpurun_out/kbm_${kb}_c.jsonl 2> gpurun_out/kbm_${kb}_c.txt
  python bench.py --steps 30 --warmup 5 --no-cpu-baseline --no-e2e > gpurun_out/kbm_bench_${kb}.json 2>/dev/null
done
unset SNP_FASTID_KBITS
paste gpurun_out/kbm_512.txt gpurun_out/kbm_1024.txt | awk -F'\t' '{print $1,$2,$3,$4,$12}'
paste gpurun_out/kbm_512_c.txt gpurun_out/kbm_1024_c.txt | awk -F'\t' '{print $1,$2,$3,$4,$12}'
for kb in 512 1024; do python -c "import json,sys; d=json.load(open(sys.argv[1])); print(sys.argv[1], d['ms_per_step'], d['roofline']['kernel_ms'], d['roofline']['frac'])" gpurun_out/kbm_bench_${kb}.json; done
