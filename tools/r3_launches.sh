# launch lists (ncu gpu__time_duration, cold-cache serialised) of one eager step per workload (TAG as $1)
T=${1:-r3l}; mkdir -p gpurun_out/$T
for w in reddit corafull_gat am_rgcn; do
  ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/$T/launch_$w.csv \
      python bench.py --workload $w --steps 1 --warmup 1 --no-e2e --no-cpu-baseline --cuda-graph off > /dev/null 2>&1
  python tools/launch_summary.py gpurun_out/$T/launch_$w.csv > gpurun_out/$T/launch_$w.txt 2>&1
done
