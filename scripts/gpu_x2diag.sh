#!/bin/bash
export SNP_LIB_PATH=$PWD/paper_conf_ipps_binderlp19_b200/libsnp_skip.so
export SNP_X2_REPORT=1
for x in 1; do for sk in 0 1; do
  SNP_GEMM_X2=$x SNP_DEBUG_SKIP_EXPAND=$sk python bench.py --workload ld32k --ld-layout rows --steps 5 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/x2.json 2>gpurun_out/x2.err
  head -2 gpurun_out/x2.err
  python -c "import json,sys; d=json.load(open(sys.argv[1])); print('x2', sys.argv[2], 'skip', sys.argv[3], d['ms_per_step'], d['roofline']['kernel_ms'])" gpurun_out/x2.json $x $sk || tail -3 gpurun_out/x2.err
done; done
