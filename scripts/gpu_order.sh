timeout 600 python -m pytest tests -m gpu -x -q -k "ld" 2>&1 | tail -1
for o in 2 1; do echo "order $o"; SNP_GEMM_ORDER=$o timeout 300 python scripts/ld_exp.py 2>&1 | tail -1; done
SNP_GEMM_ORDER=2 COUNTS=1 timeout 600 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum -k regex:gemm_tc4 -c 1 python scripts/ld_one.py 2>&1 | grep -E "dram|duration"
