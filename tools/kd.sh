# A/B dense-kernel timing of library variants: kd.sh base old s4 ... (variants/libseastar_X.so; base = in-tree)
LIB=paper_conf_eurosys_wumcjlzcy21_b200/libseastar.so
cp $LIB /tmp/libseastar_orig.so
for v in "$@"; do
  if [ "$v" != base ]; then cp variants/libseastar_$v.so $LIB; fi
  echo "== $v"; timeout 300 python tools/bench_dense.py 2>&1 | grep -v Warn
  cp /tmp/libseastar_orig.so $LIB
done
