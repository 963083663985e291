python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || true
timeout 900 python -m pytest tests -m gpu -q -x > gpurun_out/pytest_gpu.log 2>&1; tail -3 gpurun_out/pytest_gpu.log
B="python bench.py --no-e2e --no-cpu-baseline --steps 5 --warmup 3"
show() { python -c "
import json; d=json.loads(open('gpurun_out/t.log').read().strip().splitlines()[-1]); t=d['transfers']; print(round(d['value'],2), d['unit'], 'us/launch', round(d['us_per_launch'],1), 'host_us', round(d['host_us_per_launch'],2), 'moved', t['moved_bytes'], 'copies', t['copies'], 'strided', t['strided_copies'], 'replays', d['graph_replays'], 'kern', t.get('halo_copy_kernels'))" 2>&1 | tail -1; }
for cfg in "--parts 8" "--parts 8 --tiles 4x2" "--parts 8 --tiles 2x4"; do
  timeout 300 $B $cfg > gpurun_out/t.log 2>&1; echo "hotspot $cfg: $(show)"
done
for cfg in "--parts 8 --tiles 1x2x4" "--parts 8 --tiles 2x2x2"; do
  timeout 300 $B --workload heat3d $cfg > gpurun_out/t.log 2>&1; echo "heat $cfg: $(show)"
done
for cfg in "--parts 8" "--parts 8 --tiles 4x2"; do
  timeout 300 $B --workload jacobi2d $cfg > gpurun_out/t.log 2>&1; echo "jacobi $cfg: $(show)"
done
