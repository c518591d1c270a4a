# small configs: long-row policy A/B on CoraFull / Cora / Physics (TAG as $1)
T=${1:-r2sm}
mkdir -p gpurun_out/$T
timeout 300 python -m pytest tests/test_gpu_gcn.py tests/test_gpu_borders.py tests/test_gpu_partition.py tests/test_gpu_gat.py tests/test_gpu_dropout.py -q -x > gpurun_out/$T/tests.log 2>&1; echo "tests rc=$?"; tail -1 gpurun_out/$T/tests.log
for w in corafull_gat cora_gcn physics_appnp; do
  for mode in default off; do
    if [ $mode = off ]; then export SEASTAR_LONG_ROW=0; else unset SEASTAR_LONG_ROW; fi
    timeout 200 python bench.py --workload $w --no-cpu-baseline --no-e2e --steps 50 > gpurun_out/$T/bench_${w}_${mode}.json 2> /dev/null
    python -c "import json;d=json.load(open('gpurun_out/$T/bench_${w}_${mode}.json'));print('$w', '$mode', round(d['ms_per_step'],4), {k:round(v['ms'],4) for k,v in d['kernels'].items()})"
  done
done
