# quick Reddit check (TAG as $1): GAT / GCN parity incl. border degrees and full-size kernels, then the bench line
T=${1:-r2r}
mkdir -p gpurun_out/$T
timeout 300 python -m pytest tests/test_gpu_gat.py tests/test_gpu_borders.py tests/test_gpu_gcn.py tests/test_gpu_dropout.py tests/test_gpu_partition.py tests/test_gpu_models.py -q -x > gpurun_out/$T/tests.log 2>&1; echo "tests rc=$?"; tail -2 gpurun_out/$T/tests.log
timeout 400 python -m pytest tests/test_gpu_fullsize_kernels.py -q -x > gpurun_out/$T/fullsize_kernels.log 2>&1; echo "fullsize kernels rc=$?"; tail -2 gpurun_out/$T/fullsize_kernels.log
timeout 200 python bench.py --no-cpu-baseline > gpurun_out/$T/bench.json 2> gpurun_out/$T/bench.err; python -c "import json;d=json.load(open('gpurun_out/$T/bench.json'));print(d['ms_per_step'], d['config']['epoch_ms'], {k:round(v['ms'],3) for k,v in d['kernels'].items()})"
