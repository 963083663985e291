# round 2, call 81: C2 step as 25 individual graph replays (default) vs one pk_launch_sequence (PK_BENCH_SEQ=1)
for r in 1 2 3; do
  for q in 0 1; do
    PK_BENCH_SEQ=$q timeout 300 python bench.py --steps 20 --no-e2e --no-cpu-baseline --no-e3 > /tmp/b.json 2> /tmp/b.err
    tail -1 /tmp/b.json | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('seq=$q', round(d['value'],1), 'frac', round(d['roofline']['frac'],4), 'ms/step', round(d['ms_per_step'],3), 'kms', round(d['kernel_ms_avg'],4), d['clocks']['sm_mhz'], d['clocks']['reasons'])" || tail -3 /tmp/b.err
  done
done
