# same-box A/B of the long-row (hub CTA) policy: default vs SEASTAR_LONG_ROW=0 (TAG as $1)
T=${1:-r2lr}
mkdir -p gpurun_out/$T
timeout 300 python -m pytest tests/test_gpu_gcn.py tests/test_gpu_borders.py tests/test_gpu_partition.py tests/test_gpu_gat.py -q -x > gpurun_out/$T/tests.log 2>&1; echo "tests rc=$?"; tail -1 gpurun_out/$T/tests.log
for i in 1 2; do
  for mode in default off; do
    if [ $mode = off ]; then export SEASTAR_LONG_ROW=0; else unset SEASTAR_LONG_ROW; fi
    timeout 200 python bench.py --no-cpu-baseline --no-e2e --steps 20 > gpurun_out/$T/bench_${mode}_$i.json 2> /dev/null
    python -c "import json;d=json.load(open('gpurun_out/$T/bench_${mode}_$i.json'));print('$mode', $i, round(d['ms_per_step'],3), {k:round(v['ms'],3) for k,v in d['kernels'].items()})"
  done
done
unset SEASTAR_LONG_ROW
timeout 300 python tools/ablation_sweep.py 16 64 > gpurun_out/$T/ablation.log 2>&1; tail -4 gpurun_out/$T/ablation.log
