#!/bin/bash
# ncu --set full of the kernels matching REGEX in one eager bench.py step of WORKLOAD; summary + raw CSV to OUT.
# usage: tools/prof_kernels.sh WORKLOAD REGEX OUT [COUNT]
set -uo pipefail
W=$1; RX=$2; OUT=$3; C=${4:-4}
mkdir -p "$(dirname "$OUT")"
timeout 900 ncu --set full --clock-control none --import-source on -k "regex:$RX" -c "$C" -o /tmp/prof_$$ \
    python bench.py --workload "$W" --steps 1 --warmup 1 --no-e2e --no-cpu-baseline --cuda-graph off > "$OUT.log" 2>&1
python tools/ncu_summary.py /tmp/prof_$$.ncu-rep > "$OUT.txt" 2>&1
ncu -i /tmp/prof_$$.ncu-rep --page source --csv --print-source sass > "$OUT.source.csv" 2>/dev/null; gzip -f "$OUT.source.csv"
