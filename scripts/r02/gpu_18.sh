# round 2, call 18: C4 partition sweep on one B200 (virtual partitions): copies before the kernel
# (default for same-device partitions) vs streamed under it (PK_STREAM_SAME_DEVICE=1)
for P in 1 2 4 8; do
 for s in 0 1; do
  if [ $s = 1 ] && [ $P = 1 ]; then continue; fi
  if [ $s = 1 ]; then export PK_STREAM_SAME_DEVICE=1; else unset PK_STREAM_SAME_DEVICE; fi
  timeout 300 python bench.py --workload sgemm --parts $P --steps 6 --no-e2e --no-cpu-baseline --no-e3 > /tmp/s.json 2> /tmp/s.err
  tail -1 /tmp/s.json | python -c "import json,sys; d=json.loads(sys.stdin.read()); t=d['transfers']; print('sgemm P$P stream=$s', round(d['value'],1), 'TF/s', round(d['ms_per_step'],2), 'ms/step moved', t['moved_bytes'], 'streamed', t['streamed_bytes'], 'min', t['analytic_min_bytes'], d['clocks']['sm_mhz'], d['clocks']['reasons'])" || tail -3 /tmp/s.err
 done
done
