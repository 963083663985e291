# round 2, call 59: the driver's multi-GPU launch shape on ONE GPU (functional only: all ranks share
# cuda:0): torchrun with 4 and 8 ranks for C2 (pushed halos, peer-memory SPMD) and C3, and the reference
# arm under torchrun at N = 8; rc, transfers vs the analytic minimum
for n in 4 8; do
  for w in hotspot2d heat3d; do
    timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node $n --master-addr 127.0.0.1 --master-port 2956$n bench.py --gpus $n --workload $w --steps 3 --warmup 3 --no-e2e > gpurun_out/r02_59_${w}_n$n.json 2> gpurun_out/r02_59_${w}_n$n.err; rc=$?
    echo "N=$n $w rc=$rc"; tail -1 gpurun_out/r02_59_${w}_n$n.json | python -c "import json,sys; d=json.loads(sys.stdin.read()); t=d['transfers']; print('  value', round(d['value'],1), 'n_gpus', d['n_gpus'], 'halo_push', d['config'].get('halo_push'), 'pushed', t['pushed_bytes'], 'moved', t['moved_bytes'], 'min', t['analytic_min_bytes'], 'launches', d['gpu_launches'])" || tail -5 gpurun_out/r02_59_${w}_n$n.err
  done
done
timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 8 --master-addr 127.0.0.1 --master-port 29569 bench.py --impl reference --gpus 8 --steps 2 --warmup 3 > gpurun_out/r02_59_ref_n8.json 2> gpurun_out/r02_59_ref_n8.err; echo "reference N=8 rc=$?"; grep -c '^{' gpurun_out/r02_59_ref_n8.json
