#!/bin/bash
# GPU-box profiling pass (run under gpurun): the ncu launch list of bench.py (cold-cache, serialised
# per-launch times) and one `ncu --set full` capture of the top graph kernels, summarised on the box
# (the .ncu-rep stays in /tmp: gpurun_out/ is capped at 64 MiB).  Output: gpurun_out/prof_*.
# usage: tools/profile.sh [TAG] [extra bench args]
TAG=${1:-r1}; shift
mkdir -p gpurun_out
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/prof_launches_$TAG.csv \
    python bench.py --steps 2 --warmup 1 --no-e2e --no-cpu-baseline "$@" > gpurun_out/prof_bench_$TAG.log 2>&1
python tools/launch_summary.py gpurun_out/prof_launches_$TAG.csv > gpurun_out/prof_launches_$TAG.txt 2>&1
timeout 900 ncu --set full --clock-control none --import-source on \
    -k regex:"k_gat_bwd_hpl|k_gat_fwd_hpl|k_gat_bwd_h1|k_gat_fwd_h1|k_aggregate|k_gemm_tc|k_rgcn" -c 12 \
    -o /tmp/prof_$TAG python bench.py --steps 1 --warmup 0 --no-e2e --no-cpu-baseline --cuda-graph off "$@" > gpurun_out/prof_full_$TAG.log 2>&1
python tools/ncu_summary.py /tmp/prof_$TAG.ncu-rep > gpurun_out/prof_summary_$TAG.txt 2>&1
ncu -i /tmp/prof_$TAG.ncu-rep --page raw --csv > gpurun_out/prof_raw_$TAG.csv 2>/dev/null
gzip -f gpurun_out/prof_raw_$TAG.csv
