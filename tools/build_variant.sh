#!/bin/bash
# build_variant.sh NAME "-DFLAGS..." SRC.cu [SRC.cu ...] : libseastar.so with the given sources
# recompiled under extra flags, written to variants/libseastar_NAME.so (A/B timing on the GPU box
# via tools/kv.sh; not part of the product)
set -e
cd "$(dirname "$0")/.."
python -m paper_conf_eurosys_wumcjlzcy21_b200.build > /dev/null
name=$1; flags=$2; shift 2
mkdir -p variants /tmp/variant_$name
B=paper_conf_eurosys_wumcjlzcy21_b200
: > variants/$name.ptxas
pids=""
for src in "$@"; do
  nvcc -gencode arch=compute_100a,code=sm_100a -O3 -lineinfo -std=c++17 -Xcompiler -fPIC,-O2 --expt-relaxed-constexpr \
    -Xptxas -v -I include -I $B/csrc $flags -c $B/csrc/$src -o /tmp/variant_$name/$(basename $src .cu).o 2> variants/$name.$src.ptxas &
  pids="$pids $!"
done
for p in $pids; do wait $p; done
cat variants/$name.*.ptxas >> variants/$name.ptxas
objs=""
for o in $B/build/*.o; do
  if [ -f /tmp/variant_$name/$(basename $o) ]; then objs="$objs /tmp/variant_$name/$(basename $o)"; else objs="$objs $o"; fi
done
nvcc -shared -gencode arch=compute_100a,code=sm_100a -cudart static -Xcompiler -fPIC $objs -o variants/libseastar_$name.so
echo variants/libseastar_$name.so
