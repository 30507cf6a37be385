# build_alt.sh NAME SRCDIR "flags": libsnp_NAME.so from an alternate copy of csrc/ (bisection experiments)
set -e
name=$1; src=$2; flags=$3; d=/tmp/ba_$name; mkdir -p $d
for f in $src/*.cu; do
  nvcc -gencode arch=compute_100a,code=sm_100a -lineinfo -O3 -std=c++17 -Xcompiler -fPIC -cudart static $flags -c $f -o $d/$(basename $f).o 2>/dev/null &
done; wait
nvcc -gencode arch=compute_100a,code=sm_100a -shared -cudart static -o paper_conf_ipps_binderlp19_b200/libsnp_$name.so $d/*.o
