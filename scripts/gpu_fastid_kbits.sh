#!/bin/bash
# A/B: FastID kernel stage size 512 (default) vs 1024 bits (128-byte rows per TMA box)
bash scripts/build_variant.sh k1024 "-DFASTID_KBITS=1024 -DFASTID_NS=2 -DFASTID_NS32=2 -DFASTID_NP=4"
for v in base k1024; do
  if [ $v = k1024 ]; then export SNP_LIB_PATH=$PWD/paper_conf_ipps_binderlp19_b200/libsnp_k1024.so; else unset SNP_LIB_PATH; fi
  for i in 1 2; do
    python bench.py --steps 30 --warmup 5 --no-cpu-baseline --no-e2e > gpurun_out/kb_$v.json 2>/dev/null
    python -c "import json,sys; d=json.load(open(sys.argv[1])); print(sys.argv[1], d['ms_per_step'], d['roofline']['kernel_ms'], d['roofline']['frac'], d['clocks']['sm_mhz'])" gpurun_out/kb_$v.json
  done
  SNP_FASTID_STREAM=0 python scripts/sweep.py --M 8,32 --N 20000000 --K 2048,4096 --max-popc-s 0 > /dev/null 2> gpurun_out/kb_sweep_$v.txt
  cat gpurun_out/kb_sweep_$v.txt
done
