python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || true
B="python bench.py --no-e2e --no-cpu-baseline --steps 5 --warmup 3"
show() { python -c "
import json; d=json.loads(open('gpurun_out/t.log').read().strip().splitlines()[-1]); t=d['transfers']; print(round(d['value'],1), d['unit'], 'us/launch', round(d['us_per_launch'],1), 'host_us', round(d['host_us_per_launch'],2), 'moved', t['moved_bytes'], 'pushed', t['pushed_bytes'], 'copies', t['copies'], 'replays', d['graph_replays'])" 2>&1 | tail -1; }
for cfg in "--parts 8" "--parts 8 --push" "--parts 2" "--parts 2 --push"; do
  timeout 300 $B $cfg > gpurun_out/t.log 2>&1; echo "hotspot tbk $cfg: $(show)"
done
for cfg in "--parts 8" "--parts 8 --push"; do
  timeout 300 $B --workload heat3d $cfg > gpurun_out/t.log 2>&1; echo "heat $cfg: $(show)"
  timeout 300 $B --workload jacobi2d $cfg > gpurun_out/t.log 2>&1; echo "jacobi $cfg: $(show)"
done
OMP_NUM_THREADS=1 timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node=2 --master-addr=127.0.0.1 --master-port=29561 bench.py --gpus 2 --steps 3 --warmup 3 --no-e2e --push > gpurun_out/t.log 2>&1; echo "spmd2 push: $(show)"
