# A/B of k_aggregate variants on the F sweep (seastar column only matters); "base" = the in-tree library
LIB=paper_conf_eurosys_wumcjlzcy21_b200/libseastar.so
cp $LIB /tmp/libseastar_orig.so
for v in "$@"; do
  if [ "$v" != base ]; then cp variants/libseastar_$v.so $LIB; fi
  echo "== $v"; python tools/ablation_sweep.py 1 4 8 16 32 64 2>&1 | grep '^{' | python -c "
import sys, json
print(' '.join(f\"F{d['F']}:{d['seastar']:.3f}\" for d in map(json.loads, sys.stdin)))"
  cp /tmp/libseastar_orig.so $LIB
done
