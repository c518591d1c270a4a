# round-2 evidence pass (TAG as $1): full GPU suite, smoke, every workload's bench line, sanitizer, parity log
T=${1:-r2full}
mkdir -p gpurun_out/$T
SEASTAR_PARITY_LOG=gpurun_out/$T/parity_fullsize.jsonl timeout 1200 python -m pytest tests -m gpu -q > gpurun_out/$T/gputest.log 2>&1; echo "gpu tests rc=$?"; tail -2 gpurun_out/$T/gputest.log
timeout 120 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/$T/smoke.log 2>&1; echo "smoke rc=$?"; tail -1 gpurun_out/$T/smoke.log
timeout 400 python bench.py > gpurun_out/$T/bench.json 2> gpurun_out/$T/bench.err; echo "bench rc=$?"
python -c "import json;d=json.load(open('gpurun_out/$T/bench.json'));print(d['ms_per_step'], d['config']['epoch_ms'], d['e2e']['ms_per_step'], d['roofline']['kernel'], d['roofline']['frac'], d['cpu_baseline']['value'], d['cpu_baseline']['seconds'], d['gpu_launches'])"
for w in cora_gcn corafull_gat physics_appnp am_rgcn aifb_rgcnb mutag_rgcnb bgs_rgcnb; do
  timeout 300 python bench.py --workload $w > gpurun_out/$T/bench_$w.json 2> gpurun_out/$T/bench_$w.err
  python -c "import json;d=json.load(open('gpurun_out/$T/bench_$w.json'));print('$w', round(d['ms_per_step'],4), round(d['e2e']['ms_per_step'],4), round(d['cpu_baseline']['value']/1e6,3))"
done
# compute-sanitizer is closed on this pool (gpurun refuses it); r2 logs: profiles/r2/r2full1/sanitize_*.log
# bash tools/sanitize.sh gpurun_out/$T
