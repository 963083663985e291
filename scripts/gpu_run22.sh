B="python bench.py --no-e2e --no-cpu-baseline --steps 5 --warmup 3"
for cfg in "--parts 8" "--parts 8 --tiles 4x2" "--parts 8 --tiles 2x4" "--parts 8 --variant hotspot2d" "--parts 8 --variant hotspot2d --tiles 4x2"; do
  timeout 300 $B $cfg > gpurun_out/t.log 2>&1; echo "hotspot $cfg: $(python -c "
import json; d=json.loads(open('gpurun_out/t.log').read().strip().splitlines()[-1]); t=d['transfers']; print(round(d['value'],1), d['unit'], 'us/launch', round(d['us_per_launch'],1), 'host_us', round(d['host_us_per_launch'],2), 'moved', t['moved_bytes'], 'copies', t['copies'], 'strided', t['strided_copies'], 'replays', d['graph_replays'])" 2>&1 | tail -1)"
done
for cfg in "--parts 8" "--parts 8 --tiles 1x2x4" "--parts 8 --tiles 2x2x2"; do
  timeout 300 $B --workload heat3d $cfg > gpurun_out/t.log 2>&1; echo "heat $cfg: $(python -c "
import json; d=json.loads(open('gpurun_out/t.log').read().strip().splitlines()[-1]); t=d['transfers']; print(round(d['value'],1), d['unit'], 'us/launch', round(d['us_per_launch'],1), 'host_us', round(d['host_us_per_launch'],2), 'moved', t['moved_bytes'], 'copies', t['copies'], 'strided', t['strided_copies'], 'replays', d['graph_replays'])" 2>&1 | tail -1)"
done
for cfg in "--parts 8" "--parts 8 --tiles 4x2" "--parts 4 --tiles 2x2" "--parts 4"; do
  timeout 300 $B --workload jacobi2d $cfg > gpurun_out/t.log 2>&1; echo "jacobi $cfg: $(python -c "
import json; d=json.loads(open('gpurun_out/t.log').read().strip().splitlines()[-1]); t=d['transfers']; print(round(d['value'],2), d['unit'], 'us/launch', round(d['us_per_launch'],1), 'host_us', round(d['host_us_per_launch'],2), 'moved', t['moved_bytes'], 'copies', t['copies'], 'strided', t['strided_copies'], 'replays', d['graph_replays'])" 2>&1 | tail -1)"
done
