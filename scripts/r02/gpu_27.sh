# round 2, call 27: the driver's multi-GPU launch shape (torchrun, 2 ranks) on the one GPU: bench must run
# for every workload (ranks share the device; IPC peer pulls); and the reference arm under torchrun
for w in hotspot2d heat3d sgemm nbody jacobi2d; do
  st=3; [ $w = nbody ] && st=1
  timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29611 bench.py --gpus 2 --workload $w --steps $st --warmup 3 > /tmp/t.log 2> /tmp/t.err
  grep '^{' /tmp/t.log | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); t=d['transfers']; print('$w N=2', round(d['value'],1), d['unit'], 'moved', t['moved_bytes'], 'min', t['analytic_min_bytes'], 'e2e', (d.get('e2e') or {}).get('value'), d['config']['process_model'][:40], d.get('nvlink_nvml'))" || { echo "$w FAILED"; tail -5 /tmp/t.err; }
done
timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29612 bench.py --gpus 2 --impl reference --steps 2 --warmup 3 2>/dev/null | grep '^{' | cut -c1-200
