#!/bin/bash
# compute-sanitizer over scripts/sanitize.py (tiny shapes of every kernel family), each
# tool under its own timeout; logs in gpurun_out/sanitize/ (summaries go to profiles/).
mkdir -p gpurun_out/sanitize
CS=/usr/local/cuda/bin/compute-sanitizer
for tool in memcheck racecheck synccheck initcheck; do
  timeout ${SAN_TIMEOUT:-900} $CS --tool $tool --target-processes all --print-limit 50 \
     python scripts/sanitize.py > gpurun_out/sanitize/$tool.log 2>&1
  echo "$tool rc=$?" >> gpurun_out/sanitize/rc.txt
done
# the kind::i8 kernel and the CTA-pair LD kernel are selected by env (read once per process)
for tool in memcheck racecheck synccheck; do
  SNP_TC_KIND=i8 timeout ${SAN_TIMEOUT:-900} $CS --tool $tool --print-limit 50 python scripts/sanitize.py \
     > gpurun_out/sanitize/${tool}_i8.log 2>&1; echo "${tool}_i8 rc=$?" >> gpurun_out/sanitize/rc.txt
  SNP_GEMM_X2=1 timeout ${SAN_TIMEOUT:-900} $CS --tool $tool --print-limit 50 python scripts/sanitize.py \
     > gpurun_out/sanitize/${tool}_x2.log 2>&1; echo "${tool}_x2 rc=$?" >> gpurun_out/sanitize/rc.txt
done
