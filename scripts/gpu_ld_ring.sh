#!/bin/bash
# LD-32K: packed-ring depth (GEMM_NP) vs expanded slots (GEMM_NS), with and without the
# expansion skipped (is the MMA stream bound by the ring's L2 round trip?)
# (libraries built beforehand: bash scripts/build_variant.sh npXnsY "-DGEMM_DEBUG_SKIP -DGEMM_NP=X -DGEMM_NS=Y")
for v in "6 3" "8 2" "4 3"; do set -- $v
  for sk in 0 1; do for w in ld32k ld2k; do
    SNP_LIB_PATH=$PWD/paper_conf_ipps_binderlp19_b200/libsnp_np$1ns$2.so SNP_DEBUG_SKIP_EXPAND=$sk python bench.py --workload $w --steps 10 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/ring.json 2>gpurun_out/ring.err
    python -c "import json,sys; d=json.load(open(sys.argv[1])); print(sys.argv[2], d['ms_per_step'], d['roofline']['kernel_ms'], d.get('clocks',{}).get('sm_mhz'), d.get('clocks',{}).get('reasons'))" gpurun_out/ring.json "$w NP=$1 NS=$2 skip=$sk" || tail -3 gpurun_out/ring.err
  done; done
done
