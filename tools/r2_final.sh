# round-2 final evidence pass at HEAD (TAG as $1): GPU suite + smoke, every workload's bench line, cold launch
# lists, ncu --set full summaries of the top kernels (text only: the .ncu-rep files are deleted on the box to stay
# under gpurun's 64 MiB pull limit), and the per-kernel DRAM traffic bench.py reads (tools/capture_traffic.sh)
T=${1:-r2final}
O=gpurun_out/$T
mkdir -p $O
SEASTAR_PARITY_LOG=$O/parity_fullsize.jsonl timeout 1200 python -m pytest tests -m gpu -q > $O/gputest.log 2>&1; echo "gpu tests rc=$?"; tail -1 $O/gputest.log
timeout 120 python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke.log 2>&1; echo "smoke rc=$?"; tail -1 $O/smoke.log
for w in reddit am_rgcn corafull_gat physics_appnp cora_gcn; do
  bash tools/capture_traffic.sh $w $O > /dev/null 2>&1; echo "traffic $w rc=$?"
done
timeout 400 python bench.py > $O/bench.json 2> $O/bench.err; echo "bench rc=$?"
for w in cora_gcn corafull_gat physics_appnp am_rgcn aifb_rgcnb mutag_rgcnb bgs_rgcnb; do
  timeout 300 python bench.py --workload $w > $O/bench_$w.json 2> $O/bench_$w.err
done
for w in reddit am_rgcn corafull_gat; do
  ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $O/launch_$w.csv \
      python bench.py --workload $w --steps 1 --warmup 1 --no-e2e --no-cpu-baseline --cuda-graph off > /dev/null 2>&1
  python tools/launch_summary.py $O/launch_$w.csv > $O/launch_$w.txt 2>&1
  rm -f $O/launch_$w.csv
done
full() {   # full() NAME WORKLOAD REGEX
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:"$3" -c 1 -o /tmp/ncu_$1 -f \
      python bench.py --workload $2 --steps 1 --warmup 0 --no-e2e --no-cpu-baseline --cuda-graph off > /dev/null 2>&1
  ncu -i /tmp/ncu_$1.ncu-rep --page details > $O/ncu_full_$1.txt 2>&1
  ncu -i /tmp/ncu_$1.ncu-rep --page raw --csv > /tmp/raw_$1.csv 2>&1
  python - "$1" > $O/ncu_raw_$1.txt <<'PY'
import csv, sys
rows = list(csv.reader(open(f"/tmp/raw_{sys.argv[1]}.csv")))
h = rows[0]
for d in rows[2:]:
    print(d[h.index("Kernel Name")][:90])
    for m in ["gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum", "lts__t_sectors_srcunit_tex_op_read.sum",
              "lts__t_sector_hit_rate.pct", "smsp__inst_executed.sum", "sm__warps_active.avg.pct_of_peak_sustained_active",
              "l1tex__data_pipe_lsu_wavefronts_mem_shared.sum", "l1tex__data_bank_conflicts_pipe_lsu_mem_shared.sum"]:
        if m in h:
            print(f"  {m:60s} {d[h.index(m)]} {rows[1][h.index(m)]}")
    st = []
    for i, m in enumerate(h):
        if "pcsamp_warps_issue_stalled" in m and not m.endswith("not_issued"):
            try:
                st.append((float(d[i].replace(",", "")), m))
            except ValueError:
                pass
    for v, m in sorted(st, reverse=True)[:6]:
        print(f"  stall {m:58s} {v:.0f}")
PY
  rm -f /tmp/ncu_$1.ncu-rep
}
full gat_bwd1 reddit "k_gat_bwd_hpl"
full gat_fwd1 reddit "k_gat_fwd_hpl"
full aggregate reddit "k_aggregate"
full gemm_tc2 reddit "k_gemm_tc2"
full gemm_tc_tn2 reddit "k_gemm_tc_tn2"
full rgcn_tile am_rgcn "k_rgcn_tile_p"
full rgcn_dw_tile am_rgcn "k_rgcn_dw_tile"
ls -la $O
