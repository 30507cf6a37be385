#!/bin/bash
# FastID-1M A/B of cheap knobs: write-back count stores, TMA L2 promotion, 512-bit stages
bash scripts/build_variant.sh wb "-DFASTID_STORE_WB" &
bash scripts/build_variant.sh promo "-DSNP_TMA_L2_PROMO_NONE" &
wait
for v in base wb promo base k512; do
  unset SNP_LIB_PATH SNP_FASTID_KBITS
  if [ $v = wb ] || [ $v = promo ]; then export SNP_LIB_PATH=$PWD/paper_conf_ipps_binderlp19_b200/libsnp_$v.so; fi
  if [ $v = k512 ]; then export SNP_FASTID_KBITS=512; fi
  python bench.py --steps 50 --warmup 5 --no-cpu-baseline --no-e2e > gpurun_out/knob_$v.json 2>/dev/null
  python -c "import json,sys; d=json.load(open(sys.argv[1])); print(sys.argv[1], round(d['ms_per_step'],5), round(d['roofline']['kernel_ms'],5), round(d['roofline']['frac'],4), d['clocks']['sm_mhz'])" gpurun_out/knob_$v.json
done
