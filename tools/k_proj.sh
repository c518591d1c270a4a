# per-launch durations of the GAT attention-projection backward kernels (one GAT epoch, eager)
ncu --metrics gpu__time_duration.sum --clock-control none -k regex:"attn_proj_bwd" --csv python bench.py --model gat --steps 1 --warmup 0 --no-e2e --no-cpu-baseline --cuda-graph off 2>/dev/null | grep -E "attn_proj_bwd" | awk -F'","' '{print substr($5,1,40), $NF}'
