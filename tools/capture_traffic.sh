#!/bin/bash
# Per-kernel DRAM traffic and L2 hit rate of bench.py's timed graph kernels AT HEAD (run under gpurun, one GPU).
# bench.py (SEASTAR_NVTX=1) wraps its per-kernel timer pass in an NVTX range and each timed kernel in a range
# named like the JSON line's `kernels` keys; ncu renames every kernel by its innermost range, so the CSV maps
# straight onto bench.py's names.  tools/traffic_json.py writes profiles/<round>/ncu_traffic_<workload>.json with
# the source hash bench.py compares against (the numbers are only used when they were captured at this source).
# usage: tools/capture_traffic.sh WORKLOAD OUTDIR
set -euo pipefail
W=${1:-reddit}
OUT=${2:-gpurun_out}
mkdir -p "$OUT" gpurun_out
SEASTAR_NVTX=1 ncu --nvtx --print-nvtx-rename kernel --clock-control none \
    --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,lts__t_sector_hit_rate.pct,lts__t_bytes.sum \
    --csv --log-file gpurun_out/traffic_$W.csv \
    python bench.py --workload "$W" --steps 1 --warmup 1 --no-e2e --no-cpu-baseline --cuda-graph off \
    > gpurun_out/traffic_$W.log 2>&1
python tools/traffic_json.py gpurun_out/traffic_$W.csv "$W" > "$OUT/ncu_traffic_$W.json"
