# round-2 scratch pass (TAG as $1): quick parity of the changed kernels, AM + Reddit bench, AM launch list.
# Every step has its own short timeout so a hung kernel costs minutes, not the whole call.
T=${1:-r2x}
mkdir -p gpurun_out/$T
timeout 240 python -m pytest tests/test_gpu_rgcn.py tests/test_gpu_borders.py tests/test_gpu_gcn.py tests/test_gpu_gat.py -q -x > gpurun_out/$T/tests_a.log 2>&1; echo "tests_a rc=$?"; tail -3 gpurun_out/$T/tests_a.log
timeout 300 python -m pytest tests/test_gpu_models.py tests/test_gpu_rgcn_basis.py tests/test_gpu_partition.py tests/test_gpu_dense.py tests/test_gpu_dropout.py -q -x > gpurun_out/$T/tests_b.log 2>&1; echo "tests_b rc=$?"; tail -3 gpurun_out/$T/tests_b.log
timeout 150 python bench.py --workload am_rgcn --no-cpu-baseline > gpurun_out/$T/bench_am.json 2> gpurun_out/$T/bench_am.err; python -c "import json;d=json.load(open('gpurun_out/$T/bench_am.json'));print(d['ms_per_step'], d['kernels'])"
timeout 200 python bench.py --no-cpu-baseline > gpurun_out/$T/bench.json 2> gpurun_out/$T/bench.err; python -c "import json;d=json.load(open('gpurun_out/$T/bench.json'));print(d['ms_per_step'], d['config']['epoch_ms'], {k:round(v['ms'],3) for k,v in d['kernels'].items()})"
timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/$T/launches_am.csv python bench.py --workload am_rgcn --steps 2 --warmup 1 --no-e2e --no-cpu-baseline --cuda-graph off > /dev/null 2>&1; python tools/launch_summary.py gpurun_out/$T/launches_am.csv > gpurun_out/$T/launches_am.txt; head -14 gpurun_out/$T/launches_am.txt
