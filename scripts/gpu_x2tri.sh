#!/bin/bash
SNP_GEMM_X2=1 timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_exactness.py -q -x -m gpu -k "ld_sym or stream_ld_sym or ld" 2>&1 | tail -3
for rep in 1 2; do for w in ld32k ld2k; do for x in 0 1; do
  SNP_GEMM_X2=$x python bench.py --workload $w --steps 20 --warmup 5 --no-cpu-baseline --no-e2e > gpurun_out/x2t.json 2>gpurun_out/x2t.err
  python -c "import json,sys; d=json.load(open(sys.argv[1])); print(sys.argv[3], 'x2', sys.argv[2], d['ms_per_step'], d['roofline']['kernel_ms'], d['roofline']['frac'], d['clocks'])" gpurun_out/x2t.json $x $w || tail -3 gpurun_out/x2t.err
done; done; done
