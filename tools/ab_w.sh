# A/B of library variants on one workload: ab_w.sh WORKLOAD V1 V2 ... (variants/libseastar_X.so on the box)
W=$1; shift
LIB=paper_conf_eurosys_wumcjlzcy21_b200/libseastar.so
cp $LIB /tmp/libseastar_orig.so
trap 'cp /tmp/libseastar_orig.so $LIB' EXIT
for v in base "$@" base; do
  if [ $v != base ]; then cp variants/libseastar_$v.so $LIB; else cp /tmp/libseastar_orig.so $LIB; fi
  timeout 300 python bench.py --workload $W --no-cpu-baseline --no-e2e --steps 50 > /tmp/b.json 2>/dev/null
  python -c "import json;d=json.load(open('/tmp/b.json'));print('$W', '$v', round(d['ms_per_step'],4), {k:round(v['ms'],4) for k,v in d['kernels'].items()})"
done
