#!/bin/bash
bash scripts/build_variant.sh wbp "-DFASTID_STORE_WB -DSNP_TMA_L2_PROMO_NONE" &
bash scripts/build_variant.sh wb "-DFASTID_STORE_WB" &
wait
for v in wb wbp wb wbp; do
  export SNP_LIB_PATH=$PWD/paper_conf_ipps_binderlp19_b200/libsnp_$v.so
  python bench.py --steps 50 --warmup 5 --no-cpu-baseline --no-e2e > gpurun_out/knob_$v.json 2>/dev/null
  python -c "import json,sys; d=json.load(open(sys.argv[1])); print(sys.argv[1], round(d['ms_per_step'],5), round(d['roofline']['kernel_ms'],5), round(d['roofline']['frac'],4), d['clocks']['sm_mhz'])" gpurun_out/knob_$v.json
done
for v in wb wbp; do
  export SNP_LIB_PATH=$PWD/paper_conf_ipps_binderlp19_b200/libsnp_$v.so
  python bench.py --workload ld32k --steps 10 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/knob_ld_$v.json 2>/dev/null
  python -c "import json,sys; d=json.load(open(sys.argv[1])); print(sys.argv[1], round(d['ms_per_step'],5), round(d['roofline']['kernel_ms'],5), round(d['roofline']['frac'],4), d['clocks']['sm_mhz'])" gpurun_out/knob_ld_$v.json
  SNP_FASTID_STREAM=0 python scripts/sweep.py --M 8,32 --N 20000000 --K 4096 --max-popc-s 0 2>&1 >/dev/null | tail -2
done
