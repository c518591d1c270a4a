# A/B of GAT kernel variants on the Reddit bench (kernel timers; GAT model only)
LIB=paper_conf_eurosys_wumcjlzcy21_b200/libseastar.so
cp $LIB /tmp/libseastar_orig.so
for v in base "$@"; do
  if [ "$v" != base ]; then cp variants/libseastar_$v.so $LIB; fi
  echo "== $v"; python bench.py --model gat --steps 10 --no-e2e --no-cpu-baseline 2>/dev/null | python -c "
import sys, json
d = json.loads(sys.stdin.read()); print(round(d['ms_per_step'], 3), {k: round(v['ms'], 3) for k, v in d['kernels'].items()})"
  cp /tmp/libseastar_orig.so $LIB
done
