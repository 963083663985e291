# Partition sweep on one B200: P = 1, 2, 4, 8 virtual partitions (full-size instances on cuda:0), transfers
# included, with the alpha/beta/gamma overhead decomposition (section 9.2)
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || tail -5 gpurun_out/build.log
: > gpurun_out/partition_sweep.jsonl
for w in hotspot2d heat3d jacobi2d nbody sgemm; do
for P in 1 2 4 8; do
  st=5; [ $w = nbody ] && st=2; [ $w = sgemm ] && st=3
  timeout 900 python bench.py --workload $w --parts $P --abg --steps $st --warmup 3 --no-e2e --no-cpu-baseline > /tmp/b.log 2>&1
  tail -1 /tmp/b.log >> gpurun_out/partition_sweep.jsonl || true
  tail -1 /tmp/b.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); t=d['transfers']; o=d.get('overhead',{}); print('$w P=$P', round(d['value'],1), d['unit'], 'stale', t['stale_bytes'], 'moved', t['moved_bytes'], 'min', t['analytic_min_bytes'], 'host_us', round(d['host_us_per_launch'],2), 'T_app %.3f T_tr %.3f T_pat %.3f' % (o.get('T_application',0), o.get('T_transfers',0), o.get('T_patterns',0)))" || tail -3 /tmp/b.log
done
done
