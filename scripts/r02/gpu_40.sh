# round 2, call 40: C2 rows per tile for a rank's N = 8 share (2048 rows): one-round tall tiles vs the chooser's 54
run() {
  timeout 300 python bench.py --tile $1 --steps 10 --no-e2e --no-cpu-baseline --no-e3 > /tmp/b.json 2> /tmp/b.err
  tail -1 /tmp/b.json | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('rows', '$PK_BENCH_ROWS', 'TY', $1, round(d['value'],1), 'frac', round(d['roofline']['frac'],4), 'kms', round(d['kernel_ms_avg'],4), d['clocks']['sm_mhz'])" || tail -3 /tmp/b.err
}
export PK_BENCH_ROWS=2048
for r in 1 2; do
for ty in 54 41 73 114 147 171 205 256; do run $ty; done
done
export PK_BENCH_ROWS=4096
for ty in 131 108 92 73 54; do run $ty; done
unset PK_BENCH_ROWS
run 131
