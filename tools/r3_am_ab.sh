# AM R-GCN: A/B of library variants (variants/libseastar_X.so; needs variants/ on the box) + the r2 kernels
T=${1:-r3amab}; shift
mkdir -p gpurun_out/$T
LIB=paper_conf_eurosys_wumcjlzcy21_b200/libseastar.so
cp $LIB /tmp/libseastar_orig.so
trap 'cp /tmp/libseastar_orig.so $LIB' EXIT
for v in base "$@"; do
  if [ $v != base ]; then cp variants/libseastar_$v.so $LIB; else cp /tmp/libseastar_orig.so $LIB; fi
  timeout 300 python bench.py --workload am_rgcn --no-cpu-baseline --no-e2e --steps 30 > gpurun_out/$T/bench_am_$v.json 2> gpurun_out/$T/bench_am_$v.err
  python -c "import json;d=json.load(open('gpurun_out/$T/bench_am_$v.json'));print('am', '$v', round(d['ms_per_step'],4), {k:round(v['ms'],4) for k,v in d['kernels'].items()})"
done
