#!/bin/bash
# per-tile trace of the packed-triangle LD kernel at LD-32K, expansion on / skipped
export SNP_LIB_PATH=$PWD/paper_conf_ipps_binderlp19_b200/libsnp_tr4.so
for sk in 0 1 2; do echo "== skip $sk"; SNP_DEBUG_SKIP_EXPAND=$sk MODE=ld ND=32768 NBITS=16384 python scripts/trace_gemm.py; done
