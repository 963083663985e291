# a rank's C2 share at N = 8 (2048 rows): one round of tiles (TY = 171: 12 x 35 = 420 tiles <= 444 CTAs) vs 64
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || tail -5 gpurun_out/build.log
for ty in 171 64 205 128 171 64; do
PK_BENCH_ROWS=2048 timeout 300 python bench.py --tile $ty --steps 10 --warmup 3 --no-e2e --no-cpu-baseline > /tmp/b.log 2>&1; tail -1 /tmp/b.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('rows=2048 TY=$ty', round(d['value'],1), round(d['roofline']['frac'],3), round(d['kernel_ms_avg'],4), d['clocks']['sm_mhz'])" || tail -3 /tmp/b.log
done
for ty in 342 128; do
PK_BENCH_ROWS=4096 timeout 300 python bench.py --tile $ty --steps 10 --warmup 3 --no-e2e --no-cpu-baseline > /tmp/b.log 2>&1; tail -1 /tmp/b.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('rows=4096 TY=$ty', round(d['value'],1), round(d['roofline']['frac'],3), round(d['kernel_ms_avg'],4), d['clocks']['sm_mhz'])" || tail -3 /tmp/b.log
done
