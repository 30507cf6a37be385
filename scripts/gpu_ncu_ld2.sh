set -x
mkdir -p gpurun_out/prof
COUNTS=1 timeout 600 ncu --set full --clock-control none --import-source on -k regex:gemm_tc4 -s 1 -c 1 -o gpurun_out/prof/ld_r2c python scripts/ld_one.py > gpurun_out/ncu_ld3.log 2>&1; echo $?
