# N > 1 functional check on a 1-GPU box: torchrun with 2 (and 3) ranks sharing the GPU, gloo-staged collectives
mkdir -p gpurun_out
export SEASTAR_DIST_BACKEND=gloo
for w in ${WORKLOADS:-reddit am_rgcn bgs_rgcnb physics_appnp corafull_gat cora_gcn}; do
  for P in ${PS:-2 3}; do
    timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node $P --master-addr 127.0.0.1 --master-port 29533 \
      bench.py --gpus $P --steps 3 --warmup 3 --workload $w --no-cpu-baseline > gpurun_out/dist_${w}_$P.json 2> gpurun_out/dist_${w}_$P.err
    echo "$w P=$P rc=$? $(python -c "import json,sys; d=json.load(open(sys.argv[1])); print(d['ms_per_step'], d['config']['epoch_ms'])" gpurun_out/dist_${w}_$P.json 2>&1 | tail -1)"
    grep -iE "error|exception" gpurun_out/dist_${w}_$P.err | head -3
  done
done
