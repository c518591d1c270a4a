"""Summarise an ncu --set full report: key throughput, traffic, occupancy and stall metrics."""
import csv, io, subprocess, sys

KEYS = ["Duration", "DRAM Throughput", "Memory Throughput", "L2 Cache Throughput", "L1/TEX Cache Throughput",
        "Compute (SM) Throughput", "L2 Hit Rate", "L1/TEX Hit Rate", "Achieved Occupancy", "Registers Per Thread",
        "Grid Size", "Block Size", "Issued Ipc Active", "Eligible Warps Per Scheduler", "No Eligible",
        "Warp Cycles Per Issued Instruction", "Theoretical Occupancy"]


def summary(path):
    out = subprocess.run(["ncu", "-i", path, "--page", "details", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    h = rows[0]
    res = {}
    for r in rows[1:]:
        d = dict(zip(h, r))
        res.setdefault(d["Kernel Name"][:70], {})[d["Metric Name"]] = (d["Metric Value"], d["Metric Unit"])
    raw = subprocess.run(["ncu", "-i", path, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rr = list(csv.reader(io.StringIO(raw)))
    hh = rr[0]
    for r in rr[2:]:
        d = dict(zip(hh, r))
        k = d["Kernel Name"][:70]
        for m in ["dram__bytes_read.sum", "dram__bytes_write.sum", "lts__t_bytes.sum", "smsp__inst_executed.sum",
                  "l1tex__t_bytes_pipe_lsu_mem_global_op_ld.sum", "lts__t_sectors_srcunit_tex_op_read.sum"]:
            if m in d:
                res[k][m] = (d[m], rr[1][hh.index(m)])
        stalls = {m: d[m] for m in hh if m.startswith("smsp__average_warp_latency_issue_stalled") or
                  (m.startswith("smsp__warp_issue_stalled_") and m.endswith("_per_warp_active.pct"))}
        top = sorted(((float(v.replace(",", "")), m) for m, v in stalls.items() if v not in ("", "n/a")), reverse=True)[:6]
        res[k]["top_stalls"] = [(m.replace("smsp__warp_issue_stalled_", "").replace("_per_warp_active.pct", ""), v)
                                for v, m in top]
    return res


if __name__ == "__main__":
    for p in sys.argv[1:]:
        for k, m in summary(p).items():
            print(f"== {p}: {k}")
            for key in KEYS + ["dram__bytes_read.sum", "dram__bytes_write.sum", "lts__t_bytes.sum",
                               "smsp__inst_executed.sum", "l1tex__t_bytes_pipe_lsu_mem_global_op_ld.sum"]:
                if key in m:
                    print(f"   {key:45s} {m[key][0]:>16s} {m[key][1]}")
            print("   top stalls:", m.get("top_stalls"))
