#!/bin/bash
bash scripts/build_variant.sh np4 "-DGEMM_NP=4" &
bash scripts/build_variant.sh np8 "-DGEMM_NP=8" &
wait
for w in ld2k ld32k; do
for v in base np4 np8; do
  unset SNP_LIB_PATH
  if [ $v != base ]; then export SNP_LIB_PATH=$PWD/paper_conf_ipps_binderlp19_b200/libsnp_$v.so; fi
  python bench.py --workload $w --steps 10 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/lk_$v.json 2>/dev/null
  python -c "import json,sys; d=json.load(open(sys.argv[1])); print(sys.argv[2], sys.argv[1], round(d['ms_per_step']*1e3,2), round(d['roofline']['kernel_ms']*1e3,2), d['clocks']['sm_mhz'])" gpurun_out/lk_$v.json $w
done; done
