#!/bin/bash
# gpu_ab.sh OUT LIB1 LIB2 ...: interleaved A/B of scripts/ab_fastid.py (env NQ/ND/K/COUNTS) over libraries
out=$1; shift; mkdir -p gpurun_out/ab
for r in 1 2 3; do for l in "$@"; do
  SNP_LIB_PATH=$PWD/paper_conf_ipps_binderlp19_b200/$l timeout 120 python scripts/ab_fastid.py >> gpurun_out/ab/$out.jsonl 2>>gpurun_out/ab/$out.err
done; done
cat gpurun_out/ab/$out.jsonl
