# count our kernels per training epoch of every workload (ncu launch list of: graph build, 1 timed + 1 kernel-timer epoch)
mkdir -p gpurun_out
for w in ${WORKLOADS:-cora_gcn corafull_gat physics_appnp am_rgcn aifb_rgcnb bgs_rgcnb reddit}; do
  ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/cnt_$w.csv \
      python bench.py --workload $w --steps 1 --warmup 0 --no-e2e --no-cpu-baseline --cuda-graph off > /dev/null 2>&1
  python - "$w" <<'PY'
import csv, sys
w = sys.argv[1]
rows = list(csv.reader(open(f"gpurun_out/cnt_{w}.csv")))
hi = [i for i, r in enumerate(rows) if "Kernel Name" in r][0]
k = rows[hi].index("Kernel Name")
names = [r[k] for r in rows[hi + 1:]]
# epochs start at the first kernel after graph creation: the Adam step-counter increments mark epoch ends
ends = [i for i, n in enumerate(names) if "k_step_inc" in n]
ours = lambda seg: sum(1 for n in seg if "seastar::" in n or n.startswith("void seastar") or "k_" in n and "at::" not in n and "cub::" not in n)
print(w, "step_inc at", ends, "kernels per epoch (last epoch):", ours(names[ends[-3] + 2 if len(ends) >= 3 else 0: ends[-1] + 2]) if len(ends) >= 2 else None)
PY
done
