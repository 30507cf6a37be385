set -x
timeout 120 python -m pytest tests -m gpu -x -q -k "ld_r2_dprime or ld_counts_accumulate or leading" > gpurun_out/x2_small.log 2>&1; echo small=$?; tail -3 gpurun_out/x2_small.log
timeout 600 python -m pytest tests -m gpu -x -q -k "ld" > gpurun_out/x2_ld.log 2>&1; echo ld=$?; tail -3 gpurun_out/x2_ld.log
timeout 300 python scripts/ld_exp.py 2>&1 | tail -1
M=2048 K=4096 timeout 300 python scripts/ld_exp.py 2>&1 | tail -1
SNP_GEMM_X2=0 timeout 300 python scripts/ld_exp.py 2>&1 | tail -1
