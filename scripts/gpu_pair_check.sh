#!/bin/bash
timeout 1200 python -m pytest tests/test_gpu_parity.py -q -x -m gpu -k "ld_sym or pair or selfld or ld_r2" 2>&1 | tail -3
mkdir -p gpurun_out/sanitize
CS=/usr/local/cuda/bin/compute-sanitizer
for tool in memcheck racecheck synccheck; do
  SNP_GEMM_X2=1 timeout 900 $CS --tool $tool --print-limit 50 python scripts/sanitize.py > gpurun_out/sanitize/${tool}_x2.log 2>&1
  echo "${tool}_x2 rc=$?"; grep -E "ERROR SUMMARY|RACECHECK SUMMARY|SANITIZE-PASS-DONE|MISMATCH" gpurun_out/sanitize/${tool}_x2.log | head -3
done
