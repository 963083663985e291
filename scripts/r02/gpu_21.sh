# round 2, call 21: C2 rows per tile at a rank's share for N = 4 / 8; the new default (TY from the chooser)
run() {
  timeout 300 python bench.py --tile $1 --steps 5 --no-e2e --no-cpu-baseline --no-e3 > /tmp/b.json 2> /tmp/b.err
  tail -1 /tmp/b.json | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('rows', '$PK_BENCH_ROWS', 'TY', $1, round(d['value'],1), 'frac', round(d['roofline']['frac'],4), d['clocks']['sm_mhz'], d['clocks']['reasons'])" || tail -3 /tmp/b.err
}
export PK_BENCH_ROWS=2048
for ty in 54 82 54 82; do run $ty; done
export PK_BENCH_ROWS=4096
for ty in 64 108 128 108; do run $ty; done
unset PK_BENCH_ROWS
timeout 300 python bench.py --steps 10 --no-e2e --no-cpu-baseline --no-e3 > /tmp/b.json 2>/tmp/b.err; tail -1 /tmp/b.json | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('default', d['config']['rows_per_tile'], round(d['value'],1), round(d['roofline']['frac'],4), d['clocks'])"
timeout 900 python -m pytest tests/test_gpu_fullsize.py -q -x -k c2 2>&1 | tail -1
