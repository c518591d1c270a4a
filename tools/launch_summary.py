"""Summarise an ncu --metrics gpu__time_duration.sum launch list (CSV): per-kernel totals and shares."""
import csv
import sys
from collections import defaultdict


def load(path):
    rows = list(csv.reader(open(path)))
    hdr = next(i for i, r in enumerate(rows) if r and r[0] == "ID")
    h = rows[hdr]
    ki, vi, ui = h.index("Kernel Name"), h.index("Metric Value"), h.index("Metric Unit")
    out = []
    for r in rows[hdr + 1:]:
        scale = {"nsecond": 1e-6, "ns": 1e-6, "usecond": 1e-3, "us": 1e-3, "msecond": 1.0, "ms": 1.0, "second": 1e3, "s": 1e3}[r[ui]]
        out.append((r[ki], float(r[vi].replace(",", "")) * scale))
    return out


if __name__ == "__main__":
    launches = load(sys.argv[1])
    skip = int(sys.argv[2]) if len(sys.argv) > 2 else 0
    launches = launches[skip:]
    agg = defaultdict(list)
    for k, ms in launches:
        agg[k.split("(")[0][:70]].append(ms)
    tot = sum(ms for _, ms in launches)
    print(f"{len(launches)} launches, {tot:.3f} ms total (cold-cache, serialised)")
    for k, v in sorted(agg.items(), key=lambda kv: -sum(kv[1])):
        print(f"{sum(v):9.3f} ms {100 * sum(v) / tot:5.1f}%  n={len(v):3d}  {k}")
