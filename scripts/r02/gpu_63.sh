# round 2, call 63: torchrun with 2 ranks on ONE GPU for the remaining workloads (functional): C4, C5, C1
for w in sgemm nbody jacobi2d; do
  st=2; [ $w = jacobi2d ] && st=5
  timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 2963${#w} bench.py --gpus 2 --workload $w --steps $st --warmup 3 --no-e2e > gpurun_out/r02_63_$w.json 2> gpurun_out/r02_63_$w.err; rc=$?
  echo "N=2 $w rc=$rc"; tail -1 gpurun_out/r02_63_$w.json | python -c "import json,sys; d=json.loads(sys.stdin.read()); t=d['transfers']; print('  value', round(d['value'],1), d['unit'], 'halo_push', d['config'].get('halo_push'), 'moved', t['moved_bytes'], 'pushed', t['pushed_bytes'], 'streamed', t['streamed_bytes'], 'min', t['analytic_min_bytes'], 'launches', d['gpu_launches'])" || tail -5 gpurun_out/r02_63_$w.err
done
