#!/bin/bash
for sk in 1 0; do SNP_DEBUG_SKIP_EXPAND=$sk SNP_GEMM_X2=1 SNP_LIB_PATH=$PWD/paper_conf_ipps_binderlp19_b200/libsnp_tr1.so python scripts/trace_x2.py; done
SNP_GEMM_X2=1 timeout 900 python -m pytest tests -q -x -m gpu -k "x2 or pair" 2>&1 | tail -2
for x in 0 1; do
  SNP_GEMM_X2=$x python bench.py --workload ld32k --ld-layout rows --steps 10 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/x2.json 2>gpurun_out/x2.err
  python -c "import json,sys; d=json.load(open(sys.argv[1])); print('x2', sys.argv[2], d['ms_per_step'], d['roofline']['kernel_ms'], d['clocks'])" gpurun_out/x2.json $x || tail -3 gpurun_out/x2.err
done
