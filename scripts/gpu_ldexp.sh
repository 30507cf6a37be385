set -x
timeout 300 python scripts/ld_exp.py > gpurun_out/ldexp.log 2>&1; echo $?
SNP_DEBUG_SKIP_EXPAND=1 timeout 300 python scripts/ld_exp.py > gpurun_out/ldexp_skip.log 2>&1; echo $?
cat gpurun_out/ldexp*.log
