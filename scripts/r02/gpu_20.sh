# round 2, call 20: C2 rows per tile vs the persistent grid's rounds (444 CTAs): full grid and a rank's N=8 share;
# plus the new GPU tests (paper-vs-validity measured on GPU, GEMM placement vs oracle)
timeout 600 python -m pytest tests/test_gpu_parity.py -q -x -k "paper_vs_validity or placement" 2>&1 | tail -2
run() {
  timeout 300 python bench.py --tile $1 --steps 5 --no-e2e --no-cpu-baseline --no-e3 > /tmp/b.json 2> /tmp/b.err
  tail -1 /tmp/b.json | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('rows', '$PK_BENCH_ROWS', 'TY', $1, round(d['value'],1), 'frac', round(d['roofline']['frac'],4), d['clocks']['sm_mhz'], d['clocks']['reasons'])" || tail -3 /tmp/b.err
}
export PK_BENCH_ROWS=16384
for ty in 128 131 146 164 187 218 128; do run $ty; done
export PK_BENCH_ROWS=2048
for ty in 64 54 96 103 64; do run $ty; done
