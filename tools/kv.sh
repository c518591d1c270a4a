# A/B timing of library variants: kv.sh base mb3 ... (copies variants/libseastar_X.so into place)
# (needs variants/ on the box: drop the variants/ line from .gpurunignore for that call)
LIB=paper_conf_eurosys_wumcjlzcy21_b200/libseastar.so
cp $LIB /tmp/libseastar_orig.so
for v in "$@"; do cp variants/libseastar_$v.so $LIB; bash tools/kt.sh "V=$v"; done
cp /tmp/libseastar_orig.so $LIB
