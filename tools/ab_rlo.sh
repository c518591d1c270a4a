# A/B of the low-degree R-GCN row mapping (lanes per row) on the AM shape: bench timers + R-GCN parity per variant
# (needs variants/ on the box: drop the variants/ line from .gpurunignore for that call)
set -euo pipefail
LIB=paper_conf_eurosys_wumcjlzcy21_b200/libseastar.so
mkdir -p gpurun_out
for v in rlo8 rlo16; do [ -f variants/libseastar_$v.so ] || { echo "missing variants/libseastar_$v.so" >&2; exit 1; }; done
cp $LIB /tmp/libseastar_orig.so
trap 'cp /tmp/libseastar_orig.so $LIB' EXIT          # the product library is restored however the loop ends
for v in base rlo8 rlo16 base; do
  if [ $v = base ]; then cp /tmp/libseastar_orig.so $LIB; else cp variants/libseastar_$v.so $LIB; fi
  python -m pytest tests/test_gpu_rgcn.py -x -q 2>&1 | tail -1
  python bench.py --workload am_rgcn --steps 20 --no-cpu-baseline > gpurun_out/ab_$v.json 2> /dev/null
  python -c "import json,sys; d=json.load(open(sys.argv[1])); print(sys.argv[2], 'step', round(d['ms_per_step'],3), 'fwd1', round(d['kernels']['rgcn_fwd1']['ms'],4), 'bwd2', round(d['kernels']['rgcn_bwd2']['ms'],4))" gpurun_out/ab_$v.json $v
done

