#!/bin/bash
# LD-32K (packed triangle): which expander work bounds the MMA stream?  debug_skip 1 = no
# expansion at all, 2 = only the A warps on the MMA warp's sub-partition skip (their tcgen05.st
# queue behind the issued MMAs); with and without the pre-expanded column operand.
bash scripts/build_variant.sh skip "-DGEMM_DEBUG_SKIP" > /dev/null
export SNP_LIB_PATH=$PWD/paper_conf_ipps_binderlp19_b200/libsnp_skip.so
for bp in 0 1; do for sk in 0 1 2; do
  SNP_GEMM_BPRE=$bp SNP_DEBUG_SKIP_EXPAND=$sk python bench.py --workload ld32k --steps 10 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/skip_$bp$sk.json 2>gpurun_out/skip_$bp$sk.err
  python -c "import json,sys; d=json.load(open(sys.argv[1])); print('bpre', sys.argv[2], 'skip', sys.argv[3], d['ms_per_step'], d['roofline']['kernel_ms'], d.get('clocks'))" gpurun_out/skip_$bp$sk.json $bp $sk || tail -3 gpurun_out/skip_$bp$sk.err
done; done
