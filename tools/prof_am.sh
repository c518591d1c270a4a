# AM-shaped R-GCN on the GPU box: launch list of one epoch and an ncu full capture of the layer-1 forward
# row kernels (hub, split and low-degree buckets: the first three k_rgcn_rows launches)
mkdir -p gpurun_out
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launch_am.csv \
    python bench.py --workload am_rgcn --steps 2 --warmup 1 --no-e2e --no-cpu-baseline --cuda-graph off > /dev/null 2>&1
python tools/launch_summary.py gpurun_out/launch_am.csv > gpurun_out/launch_am.txt 2>&1; head -24 gpurun_out/launch_am.txt
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_rgcn_rows -c 3 -o gpurun_out/ncu_am_rows -f \
    python bench.py --workload am_rgcn --steps 1 --warmup 0 --no-e2e --no-cpu-baseline --cuda-graph off > gpurun_out/ncu_am.log 2>&1
echo NCU_EXIT $?
