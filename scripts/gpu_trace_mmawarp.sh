#!/bin/bash
bash scripts/build_variant.sh tr2 "-DFASTID_TRACE2"
bash scripts/build_variant.sh tr2m "-DFASTID_TRACE2 -DFASTID_MMA_FIRST"
for v in tr2 tr2m; do
  export SNP_LIB_PATH=$PWD/paper_conf_ipps_binderlp19_b200/libsnp_$v.so
  MODE=bestonly NQ=1 python scripts/trace_fastid2.py > gpurun_out/trace_${v}_best1.txt 2>&1
  MODE=search NQ=64 python scripts/trace_fastid2.py > gpurun_out/trace_${v}_search64.txt 2>&1
done
unset SNP_LIB_PATH
