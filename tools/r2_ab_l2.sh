# same-box A/B: L2 persisting window on / off, repeated (TAG as $1)
T=${1:-r2ab}
mkdir -p gpurun_out/$T
for i in 1 2; do
  for mode in on off; do
    if [ $mode = on ]; then export SEASTAR_L2_PERSIST=1; else unset SEASTAR_L2_PERSIST; fi
    timeout 200 python bench.py --no-cpu-baseline --no-e2e --steps 20 > gpurun_out/$T/bench_${mode}_$i.json 2> /dev/null
    python -c "import json;d=json.load(open('gpurun_out/$T/bench_${mode}_$i.json'));print('$mode', $i, round(d['ms_per_step'],3), {k:round(v['ms'],3) for k,v in d['kernels'].items()}, d['clocks'])"
  done
done
