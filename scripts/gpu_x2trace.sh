#!/bin/bash
export SNP_LIB_PATH=$PWD/paper_conf_ipps_binderlp19_b200/libsnp_tr4.so
for x in 0 1; do for sk in 0 1; do echo "== x2 $x skip $sk"; SNP_GEMM_X2=$x SNP_DEBUG_SKIP_EXPAND=$sk MODE=ldrows ND=16384 NBITS=16384 python scripts/trace_gemm.py; done; done
