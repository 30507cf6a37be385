#!/bin/bash
# A/B on the configs[3] counts pass: early accumulator release in the swapped epilogue on/off
bash scripts/build_variant.sh noer "-DGEMM_SWAP_EARLY_RELEASE=0"
sed -n '1,100p' scripts/gpu_f20m_order.sh | sed -n '/cat > \/tmp\/f20.py/,/^PY$/p' | sed '1d;$d' > /tmp/f20.py
for v in base noer base noer; do
  unset SNP_LIB_PATH
  if [ $v = noer ]; then export SNP_LIB_PATH=$PWD/paper_conf_ipps_binderlp19_b200/libsnp_$v.so; fi
  echo -n "$v "; python /tmp/f20.py
done
