#!/bin/bash
# LD-32K: cost of the B half of the packed ring (debug_skip 3) vs baseline
export SNP_LIB_PATH=$PWD/paper_conf_ipps_binderlp19_b200/libsnp_skip.so
for sk in 0 3 0 3; do
  SNP_DEBUG_SKIP_EXPAND=$sk python bench.py --workload ld32k --steps 10 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/s3.json 2>gpurun_out/s3.err
  python -c "import json,sys; d=json.load(open(sys.argv[1])); print('skip', sys.argv[2], d['ms_per_step'], d['roofline']['kernel_ms'], d.get('clocks',{}).get('sm_mhz'), d.get('clocks',{}).get('reasons'))" gpurun_out/s3.json $sk || tail -3 gpurun_out/s3.err
done
export SNP_LIB_PATH=$PWD/paper_conf_ipps_binderlp19_b200/libsnp_tr4.so
SNP_DEBUG_SKIP_EXPAND=3 MODE=ld ND=32768 NBITS=16384 python scripts/trace_gemm.py
