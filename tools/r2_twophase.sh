# A/B of the opt-in two-phase R-GCN path on the AM shape (TAG as $1)
T=${1:-r2tp}
mkdir -p gpurun_out/$T
timeout 200 python -m pytest tests/test_gpu_rgcn.py -q -x > gpurun_out/$T/tests.log 2>&1; echo "tests rc=$?"; tail -2 gpurun_out/$T/tests.log
SEASTAR_RGCN_TWOPHASE=1 timeout 150 python bench.py --workload am_rgcn --no-cpu-baseline --no-e2e > gpurun_out/$T/bench_am_tp.json 2>&1; python -c "import json;d=json.load(open('gpurun_out/$T/bench_am_tp.json'));print('twophase', d['ms_per_step'], d['kernels'])"
SEASTAR_RGCN_TWOPHASE=1 timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/$T/launches_tp.csv python bench.py --workload am_rgcn --steps 2 --warmup 1 --no-e2e --no-cpu-baseline --cuda-graph off > /dev/null 2>&1; python tools/launch_summary.py gpurun_out/$T/launches_tp.csv > gpurun_out/$T/launches_tp.txt; head -10 gpurun_out/$T/launches_tp.txt
