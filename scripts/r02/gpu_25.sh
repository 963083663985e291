# round 2, call 25: partition sweep on one B200 (P virtual partitions, transfers included) with the
# alpha/beta/gamma decomposition as medians over 3 interleaved repeats, round-2 kernels and timing
: > gpurun_out/r02_partition_sweep.jsonl
for w in hotspot2d heat3d jacobi2d nbody sgemm; do
for P in 1 2 4 8; do
  st=5; [ $w = nbody ] && st=2; [ $w = sgemm ] && st=3
  timeout 900 python bench.py --workload $w --parts $P --abg --steps $st --warmup 3 --no-e2e --no-cpu-baseline --no-e3 > /tmp/b.log 2>&1
  tail -1 /tmp/b.log >> gpurun_out/r02_partition_sweep.jsonl || true
  tail -1 /tmp/b.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); t=d['transfers']; o=d.get('overhead',{}); sp=o.get('spread',{}); print('$w P=$P', round(d['value'],1), d['unit'], 'stale', t['stale_bytes'], 'moved', t['moved_bytes'], 'min', t['analytic_min_bytes'], 'host_us', round(d['host_us_per_launch'],2), 'T_app %.3f T_tr %.3f %s T_pat %.3f %s' % (o.get('T_application',0), o.get('T_transfers',0), [round(x,3) for x in sp.get('T_transfers',[])], o.get('T_patterns',0), [round(x,3) for x in sp.get('T_patterns',[])]))" || tail -3 /tmp/b.log
done
done
