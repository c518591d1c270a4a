# R-GCN workloads on the GPU box: parity (kernel, model, full size), bench lines, launch list of one bgs step
mkdir -p gpurun_out
python -m pytest tests/test_gpu_rgcn.py tests/test_gpu_rgcn_basis.py tests/test_gpu_models.py -x -q > gpurun_out/t_rgcn.log 2>&1; tail -2 gpurun_out/t_rgcn.log
python -m pytest tests/test_gpu_fullsize.py -k "rgcn" -x -q -s > gpurun_out/t_rgcn_full.log 2>&1; grep -E "passed|failed|rel errors" gpurun_out/t_rgcn_full.log | cut -c1-250
for w in am_rgcn aifb_rgcnb mutag_rgcnb bgs_rgcnb; do python bench.py --workload $w --steps 20 > gpurun_out/bench_$w.json 2> gpurun_out/bench_$w.err; python -c "import json,sys; d=json.load(open(sys.argv[1])); print(sys.argv[1], d['ms_per_step'], d['e2e']['ms_per_step'], d['kernels'], d['cpu_baseline']['value'])" gpurun_out/bench_$w.json; tail -3 gpurun_out/bench_$w.err; done
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launch_bgs.csv python bench.py --workload bgs_rgcnb --steps 2 --warmup 1 --no-e2e --no-cpu-baseline --cuda-graph off > /dev/null 2>&1
python tools/launch_summary.py gpurun_out/launch_bgs.csv > gpurun_out/launch_bgs.txt 2>&1; head -24 gpurun_out/launch_bgs.txt
