set -x
timeout 300 python scripts/fastid_exp.py > gpurun_out/fexp.log 2>&1; echo $?
SNP_DEBUG_NOSTORE=1 timeout 300 python scripts/fastid_exp.py > gpurun_out/fexp_nostore.log 2>&1; echo $?
cat gpurun_out/fexp*.log
