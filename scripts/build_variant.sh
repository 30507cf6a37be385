# build_variant.sh NAME "extra nvcc flags": libsnp_NAME.so next to libsnp.so (experiments)
set -e
name=$1; flags=$2; d=/tmp/bv_$name; mkdir -p $d
for f in paper_conf_ipps_binderlp19_b200/csrc/*.cu; do
  nvcc -DSNP_PROFILING -gencode arch=compute_100a,code=sm_100a -lineinfo -O3 -std=c++17 -Xcompiler -fPIC -cudart static $flags -c $f -o $d/$(basename $f).o 2>/dev/null &
done; wait
nvcc -DSNP_PROFILING -gencode arch=compute_100a,code=sm_100a -shared -cudart static -o paper_conf_ipps_binderlp19_b200/libsnp_$name.so $d/*.o
