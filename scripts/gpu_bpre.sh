#!/bin/bash
# A/B: pre-expanded column operand (SNP_GEMM_BPRE=1) vs on-chip expansion on the packed-triangle
# self-LD, plus the CTA-pair kernel on the row layout; parity of the BPRE path first.
SNP_GEMM_BPRE=1 timeout 600 python -m pytest tests/test_gpu_parity.py -q -x -m gpu -k "ld_sym or stream_ld_sym" 2>&1 | tail -3
SNP_GEMM_BPRE=1 timeout 600 python -m pytest tests/test_gpu_exactness.py -q -x -m gpu -k "ld" 2>&1 | tail -3
run() {  # tag, env..., -- bench args
  local tag=$1; shift
  local e=(); while [ "$1" != "--workload" ]; do e+=("$1"); shift; done; env "${e[@]}" python bench.py --steps 20 --warmup 5 --no-cpu-baseline --no-e2e "$@" > gpurun_out/bpre_$tag.json 2>gpurun_out/bpre_$tag.err
  python -c "import json,sys; d=json.load(open(sys.argv[1])); print(sys.argv[2], d['ms_per_step'], d['roofline']['kernel_ms'], d['roofline']['frac'], d.get('clocks'))" gpurun_out/bpre_$tag.json $tag || tail -3 gpurun_out/bpre_$tag.err
}
for rep in 1 2; do
run ld32k_base_$rep SNP_GEMM_BPRE=0 --workload ld32k
run ld32k_bpre_$rep SNP_GEMM_BPRE=1 --workload ld32k
run ld2k_base_$rep SNP_GEMM_BPRE=0 --workload ld2k
run ld2k_bpre_$rep SNP_GEMM_BPRE=1 --workload ld2k
done
run ld32k_rows SNP_GEMM_X2=0 --workload ld32k --ld-layout rows
run ld32k_rows_x2 SNP_GEMM_X2=1 --workload ld32k --ld-layout rows
