# A/B of k_aggregate variants on the F sweep (seastar column only matters)
LIB=paper_conf_eurosys_wumcjlzcy21_b200/libseastar.so
cp $LIB /tmp/libseastar_orig.so
for v in base "$@"; do
  if [ "$v" != base ]; then cp variants/libseastar_$v.so $LIB; fi
  echo "== $v"; python tools/ablation_sweep.py 1 2 4 8 16 32 2>&1 | grep '^{' | python -c "
import sys, json
for l in sys.stdin:
    d = json.loads(l); print(d['F'], round(d['seastar'], 3))"
  cp /tmp/libseastar_orig.so $LIB
done
