#!/bin/bash
bash scripts/build_variant.sh tg2 "-DFASTID_TILE_GROUP=2" &
bash scripts/build_variant.sh tg4 "-DFASTID_TILE_GROUP=4" &
wait
for v in base tg2 tg4 base tg2 tg4; do
  unset SNP_LIB_PATH
  if [ $v != base ]; then export SNP_LIB_PATH=$PWD/paper_conf_ipps_binderlp19_b200/libsnp_$v.so; fi
  python bench.py --steps 50 --warmup 5 --no-cpu-baseline --no-e2e > gpurun_out/knob_$v.json 2>/dev/null
  python -c "import json,sys; d=json.load(open(sys.argv[1])); print(sys.argv[1], round(d['ms_per_step'],5), round(d['roofline']['kernel_ms'],5), round(d['roofline']['frac'],4), d['clocks']['sm_mhz'])" gpurun_out/knob_$v.json
done
