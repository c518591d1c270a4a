# last evidence pass at the final sources (TAG as $1): GPU suite, smoke, ncu DRAM traffic of every workload (what
# bench.py's dram_frac reads), and the bench lines of the headline and the AM / CoraFull workloads
T=${1:-r2last}
O=gpurun_out/$T
mkdir -p $O
SEASTAR_PARITY_LOG=$O/parity_fullsize.jsonl timeout 1200 python -m pytest tests -m gpu -q > $O/gputest.log 2>&1; echo "gpu tests rc=$?"; tail -1 $O/gputest.log
timeout 120 python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke.log 2>&1; echo "smoke rc=$?"; tail -1 $O/smoke.log
for w in reddit am_rgcn corafull_gat physics_appnp cora_gcn; do
  bash tools/capture_traffic.sh $w $O > /dev/null 2>&1; echo "traffic $w rc=$?"
done
mkdir -p profiles/r2 && cp $O/ncu_traffic_*.json profiles/r2/
for w in reddit am_rgcn corafull_gat; do
  timeout 400 python bench.py --workload $w > $O/bench_$w.json 2> $O/bench_$w.err; echo "bench $w rc=$?"
done
