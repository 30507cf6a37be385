#!/bin/bash
# compute-sanitizer over scripts/sanitize.py with the default kernels (the four tools)
mkdir -p gpurun_out/sanitize
CS=/usr/local/cuda/bin/compute-sanitizer
for tool in memcheck racecheck synccheck initcheck; do
  timeout ${SAN_TIMEOUT:-900} $CS --tool $tool --target-processes all --print-limit 50 \
     python scripts/sanitize.py > gpurun_out/sanitize/$tool.log 2>&1
  echo "$tool rc=$?" >> gpurun_out/sanitize/rc.txt
  tail -2 gpurun_out/sanitize/$tool.log
done
