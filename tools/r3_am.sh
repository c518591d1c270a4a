# AM R-GCN tile path: parity (kernel + model + full-size step), A/B against the r2 kernels, launch list (TAG as $1)
T=${1:-r3am}
mkdir -p gpurun_out/$T
timeout 600 python -m pytest tests/test_gpu_rgcn.py tests/test_gpu_models.py -q -x -k "rgcn" > gpurun_out/$T/tests.log 2>&1; echo "tests rc=$?"; tail -3 gpurun_out/$T/tests.log
timeout 600 python -m pytest tests/test_gpu_fullsize.py -q -x -k "am_rgcn" > gpurun_out/$T/tests_full.log 2>&1; echo "full rc=$?"; tail -2 gpurun_out/$T/tests_full.log
for mode in tile standalone old; do
  unset SEASTAR_RGCN_ROWS SEASTAR_RGCN_DWG SEASTAR_RGCN_TILE_STANDALONE
  if [ $mode = old ]; then export SEASTAR_RGCN_ROWS=1 SEASTAR_RGCN_DWG=1; fi
  if [ $mode = standalone ]; then export SEASTAR_RGCN_TILE_STANDALONE=1; fi
  timeout 300 python bench.py --workload am_rgcn --no-cpu-baseline --no-e2e --steps 30 > gpurun_out/$T/bench_am_${mode}.json 2> gpurun_out/$T/bench_am_${mode}.err
  python -c "import json;d=json.load(open('gpurun_out/$T/bench_am_${mode}.json'));print('am', '$mode', round(d['ms_per_step'],4), {k:round(v['ms'],4) for k,v in d['kernels'].items()})"
done
unset SEASTAR_RGCN_ROWS SEASTAR_RGCN_DWG SEASTAR_RGCN_TILE_STANDALONE
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/$T/launch_am.csv \
    python bench.py --workload am_rgcn --steps 2 --warmup 1 --no-e2e --no-cpu-baseline --cuda-graph off > /dev/null 2>&1
python tools/launch_summary.py gpurun_out/$T/launch_am.csv > gpurun_out/$T/launch_am.txt 2>&1; head -24 gpurun_out/$T/launch_am.txt
