"""ncu CSV (tools/capture_traffic.sh) -> per-kernel traffic JSON keyed by bench.py's kernel names.

Each bench name may cover several launches (degree buckets); their bytes and times are summed.  The record
carries the source hash of libseastar.so's sources (bench.lib_src_sha) so bench.py only uses it at that source."""
import csv
import json
import os
import sys
from collections import defaultdict

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import bench  # noqa: E402


def main(path, workload):
    rows = list(csv.reader(open(path)))
    hdr = next(i for i, r in enumerate(rows) if r and r[0] == "ID")
    h = rows[hdr]
    ki, mi, vi, ui = (h.index(c) for c in ("Kernel Name", "Metric Name", "Metric Value", "Metric Unit"))
    per_launch = defaultdict(dict)
    names = {}
    for r in rows[hdr + 1:]:
        if len(r) <= vi:
            continue
        lid = int(r[0])
        names[lid] = r[ki]
        v = float(r[vi].replace(",", "")) if r[vi] not in ("", "n/a") else 0.0
        unit = r[ui]
        scale = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "nsecond": 1e-6, "ns": 1e-6, "usecond": 1e-3,
                 "us": 1e-3, "msecond": 1.0, "ms": 1.0, "%": 1.0}.get(unit, 1.0)
        per_launch[lid][r[mi]] = v * scale
    out = defaultdict(lambda: {"launches": 0, "dram_bytes": 0.0, "lts_bytes": 0.0, "ncu_ms": 0.0, "_hit": 0.0})
    for lid, m in sorted(per_launch.items()):
        # --print-nvtx-rename kernel: "<innermost range>/<kernel signature>"; bench's names carry no "::"
        head = names[lid].split("/")[0] if "/" in names[lid] else ""
        if not head or head == "seastar_timed" or "::" in head or " " in head:
            continue          # kernels outside a named range (graph creation, the rest of the timer pass)
        name = head
        o = out[name]
        o["launches"] += 1
        o["dram_bytes"] += m.get("dram__bytes_read.sum", 0) + m.get("dram__bytes_write.sum", 0)
        o["lts_bytes"] += m.get("lts__t_bytes.sum", 0)
        o["ncu_ms"] += m.get("gpu__time_duration.sum", 0)
        o["_hit"] += m.get("lts__t_sector_hit_rate.pct", 0) * m.get("lts__t_bytes.sum", 0)
    res = {}
    for k, o in out.items():
        o["l2_hit_pct"] = o.pop("_hit") / o["lts_bytes"] if o["lts_bytes"] else None
        res[k] = o
    print(json.dumps({"workload": workload, "src_sha256": bench.lib_src_sha(), "kernels": res,
                      "how": "ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,lts__t_bytes.sum,"
                             "lts__t_sector_hit_rate.pct,gpu__time_duration.sum --clock-control none over one eager "
                             "bench.py step (tools/capture_traffic.sh); bytes per bench kernel name (summed over its "
                             "bucket launches); ncu_ms is cold-cache and serialised"}, indent=1))


if __name__ == "__main__":
    main(sys.argv[1], sys.argv[2])
