#!/bin/bash
# clock64 pipeline traces of the FastID kernel (CTA 0) for the headline and a skinny shape
bash scripts/build_variant.sh tr2 "-DFASTID_TRACE2"
export SNP_LIB_PATH=$PWD/paper_conf_ipps_binderlp19_b200/libsnp_tr2.so
MODE=search NQ=64 python scripts/trace_fastid2.py > gpurun_out/trace_search64.txt 2>&1
MODE=bestonly NQ=1 python scripts/trace_fastid2.py > gpurun_out/trace_best1.txt 2>&1
MODE=bestonly NQ=32 ND=4000000 NBITS=2048 python scripts/trace_fastid2.py > gpurun_out/trace_best32_2048.txt 2>&1
