#!/bin/bash
bash scripts/build_variant.sh wb "-DGEMM_STORE_WB"
for w in ld2k ld32k; do
  for v in base wb; do
    if [ $v = wb ]; then export SNP_LIB_PATH=$PWD/paper_conf_ipps_binderlp19_b200/libsnp_wb.so; else unset SNP_LIB_PATH; fi
    python bench.py --workload $w --steps 20 --warmup 5 --no-cpu-baseline --no-e2e > gpurun_out/wb_${w}_$v.json 2>/dev/null
    python -c "import json,sys; d=json.load(open(sys.argv[1])); print(sys.argv[1], d['ms_per_step'], d['roofline']['kernel_ms'])" gpurun_out/wb_${w}_$v.json
  done
done
