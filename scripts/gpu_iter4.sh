set -x
timeout 900 python -m pytest tests -m gpu -x -q -k "ld or LD or leading" > gpurun_out/pytest_ld.log 2>&1; echo pytest=$?; tail -n 3 gpurun_out/pytest_ld.log
timeout 300 python scripts/ld_exp.py > gpurun_out/ldexp.log 2>&1
SNP_DEBUG_SKIP_EXPAND=1 timeout 300 python scripts/ld_exp.py > gpurun_out/ldexp_skip.log 2>&1
M=2048 K=4096 timeout 300 python scripts/ld_exp.py > gpurun_out/ldexp2k.log 2>&1; echo $?
for f in gpurun_out/ldexp*.log; do echo $f; cat $f; done
