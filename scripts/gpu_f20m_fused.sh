#!/bin/bash
# FastID-20M (configs[3] on 1 GPU): fused best in the general kernel's epilogue vs the previous
# library (best_reduce passes), plus the GPU tests of the changed paths
mkdir -p gpurun_out/f20
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "general_kernel_fused_best or search or ties or cfg2_search" 2>&1 | tail -3
for l in libsnp.so libsnp_old.so; do
  SNP_LIB_PATH=$PWD/paper_conf_ipps_binderlp19_b200/$l timeout 900 python bench.py --workload fastid20m --steps 5 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/f20/bench_$l.json 2>gpurun_out/f20/bench_$l.err
  python -c "
import json; d=json.loads(open('gpurun_out/f20/bench_$l.json').readline()); print('$l', d['ms_per_step'], d['roofline']['kernel_ms'], d['roofline']['frac'], d['clocks'])"
done
