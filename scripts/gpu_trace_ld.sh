#!/bin/bash
bash scripts/build_variant.sh t3 "-DGEMM_TRACE3"
SNP_LIB_PATH=$PWD/paper_conf_ipps_binderlp19_b200/libsnp_t3.so python scripts/trace_ld.py > gpurun_out/trace_ld2k.txt 2>&1
SNP_LIB_PATH=$PWD/paper_conf_ipps_binderlp19_b200/libsnp_t3.so M=32768 NBITS=16384 python scripts/trace_ld.py > gpurun_out/trace_ld32k.txt 2>&1
