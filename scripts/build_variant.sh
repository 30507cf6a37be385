# build_variant.sh NAME "extra nvcc flags": libsnp_NAME.so next to libsnp.so (experiments).
# -DSNP_PROFILING (trace hooks) unless PROF=0 (a product-equivalent build for A/B timing).
set -e
name=$1; flags=$2; d=/tmp/bv_$name; mkdir -p $d
prof=-DSNP_PROFILING; [ "${PROF:-1}" = "0" ] && prof=
for f in paper_conf_ipps_binderlp19_b200/csrc/*.cu; do
  nvcc $prof -gencode arch=compute_100a,code=sm_100a -lineinfo -O3 -std=c++17 -Xcompiler -fPIC -cudart static $flags -c $f -o $d/$(basename $f).o 2>/dev/null &
done; wait
nvcc $prof -gencode arch=compute_100a,code=sm_100a -shared -cudart static -o paper_conf_ipps_binderlp19_b200/libsnp_$name.so $d/*.o
