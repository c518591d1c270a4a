#!/bin/bash
# build_variant.sh NAME SRC.cu "-DFLAGS..." : libseastar.so with one source recompiled under extra flags,
# written to variants/libseastar_NAME.so (for A/B timing on the GPU box; not part of the product)
set -e
cd "$(dirname "$0")/.."
python -m paper_conf_eurosys_wumcjlzcy21_b200.build > /dev/null
name=$1; src=$2; flags=$3
mkdir -p variants /tmp/variant_$name
B=paper_conf_eurosys_wumcjlzcy21_b200
nvcc -gencode arch=compute_100a,code=sm_100a -O3 -lineinfo -std=c++17 -Xcompiler -fPIC,-O2 --expt-relaxed-constexpr \
  -Xptxas -v -I include -I $B/csrc $flags -c $B/csrc/$src -o /tmp/variant_$name/$(basename $src .cu).o 2> variants/$name.ptxas
objs=""
for o in $B/build/*.o; do
  if [ "$(basename $o)" == "$(basename $src .cu).o" ]; then objs="$objs /tmp/variant_$name/$(basename $o)"; else objs="$objs $o"; fi
done
nvcc -shared -gencode arch=compute_100a,code=sm_100a -cudart static -Xcompiler -fPIC $objs -o variants/libseastar_$name.so
echo variants/libseastar_$name.so
