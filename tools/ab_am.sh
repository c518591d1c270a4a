# R-GCN row-kernel change on the GPU box: R-GCN parity (kernel, model, full size), the AM bench line, launch list
mkdir -p gpurun_out
python -m pytest tests/test_gpu_rgcn.py tests/test_gpu_models.py -x -q > gpurun_out/t_rgcn.log 2>&1; tail -2 gpurun_out/t_rgcn.log
python -m pytest tests/test_gpu_fullsize.py -k "rgcn" -x -q > gpurun_out/t_rgcn_full.log 2>&1; tail -2 gpurun_out/t_rgcn_full.log
python bench.py --workload am_rgcn --steps 20 > gpurun_out/bench_am.json 2> gpurun_out/bench_am.err
python -c "import json,sys; d=json.load(open(sys.argv[1])); print(d['ms_per_step'], d['e2e']['ms_per_step'], d['kernels'], d['roofline']['frac'])" gpurun_out/bench_am.json
bash tools/prof_am.sh
