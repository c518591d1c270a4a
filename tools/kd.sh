# A/B dense-kernel timing of library variants: kd.sh base old s4 ... (variants/libseastar_X.so; base = in-tree)
# (needs variants/ on the box: drop the variants/ line from .gpurunignore for that call)
set -uo pipefail
LIB=paper_conf_eurosys_wumcjlzcy21_b200/libseastar.so
for v in "$@"; do [ "$v" = base ] || [ -f variants/libseastar_$v.so ] || { echo "missing variants/libseastar_$v.so" >&2; exit 1; }; done
cp $LIB /tmp/libseastar_orig.so
trap 'cp /tmp/libseastar_orig.so $LIB' EXIT          # the product library is restored however the loop ends
for v in "$@"; do
  if [ "$v" != base ]; then cp variants/libseastar_$v.so $LIB; fi
  echo "== $v"; timeout 300 python tools/bench_dense.py 2>&1 | grep -v Warn
  cp /tmp/libseastar_orig.so $LIB
done
