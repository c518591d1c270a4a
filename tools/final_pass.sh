# round-end evidence on one GPU box: full GPU suite, smoke, bench line, ncu launch list, ncu full of the dominant kernel
TAG=${1:-r1d}
mkdir -p gpurun_out
python -m pytest tests -m gpu -q > gpurun_out/gputest_$TAG.log 2>&1; tail -1 gpurun_out/gputest_$TAG.log
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke_$TAG.log 2>&1; tail -1 gpurun_out/smoke_$TAG.log
python bench.py > gpurun_out/bench_$TAG.json 2> gpurun_out/bench_$TAG.err; python -c "import json,sys; d=json.load(open(sys.argv[1])); print(d['ms_per_step'], d['config']['epoch_ms'], d['e2e']['ms_per_step'], d['roofline'])" gpurun_out/bench_$TAG.json
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_$TAG.csv \
    python bench.py --steps 2 --warmup 1 --no-e2e --no-cpu-baseline > /dev/null 2>&1
python tools/launch_summary.py gpurun_out/launches_$TAG.csv > gpurun_out/launches_$TAG.txt 2>&1; head -12 gpurun_out/launches_$TAG.txt
timeout 600 ncu --set full --clock-control none --import-source on -k regex:"k_gat_bwd_hpl|k_gat_fwd_hpl|k_aggregate" -c 3 \
    -o /tmp/full_$TAG python bench.py --steps 1 --warmup 0 --no-e2e --no-cpu-baseline --cuda-graph off > gpurun_out/ncu_full_$TAG.log 2>&1
python tools/ncu_summary.py /tmp/full_$TAG.ncu-rep > gpurun_out/ncu_full_$TAG.txt 2>&1; grep -E "==|Duration|dram__bytes" gpurun_out/ncu_full_$TAG.txt
