# A/B timing of library variants: kv.sh base mb3 ... (copies variants/libseastar_X.so into place)
# (needs variants/ on the box: drop the variants/ line from .gpurunignore for that call)
set -euo pipefail
LIB=paper_conf_eurosys_wumcjlzcy21_b200/libseastar.so
for v in "$@"; do [ -f variants/libseastar_$v.so ] || { echo "missing variants/libseastar_$v.so" >&2; exit 1; }; done
cp $LIB /tmp/libseastar_orig.so
trap 'cp /tmp/libseastar_orig.so $LIB' EXIT          # the product library is restored however the loop ends
for v in "$@"; do cp variants/libseastar_$v.so $LIB; bash tools/kt.sh "V=$v"; done
