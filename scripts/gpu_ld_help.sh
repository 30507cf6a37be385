#!/bin/bash
bash scripts/build_variant.sh nohelp "-DGEMM_EPI_HELP=0"
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "ld or sym or fuzz or leading or unaligned" > gpurun_out/ldh.txt 2>&1; tail -2 gpurun_out/ldh.txt
for w in ld2k ld32k; do
for v in base nohelp base nohelp; do
  unset SNP_LIB_PATH
  if [ $v = nohelp ]; then export SNP_LIB_PATH=$PWD/paper_conf_ipps_binderlp19_b200/libsnp_$v.so; fi
  python bench.py --workload $w --steps 20 --warmup 5 --no-cpu-baseline --no-e2e > gpurun_out/h_$v.json 2>/dev/null
  python -c "import json,sys; d=json.load(open(sys.argv[1])); print(sys.argv[2], sys.argv[1], round(d['ms_per_step']*1e3,2), round(d['roofline']['kernel_ms']*1e3,2), d['clocks']['sm_mhz'])" gpurun_out/h_$v.json $w
done; done
