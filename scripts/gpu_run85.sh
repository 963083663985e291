# hotspot2d_tbk with per-CTA runs (one tall tile per column segment): parity, then N = 1 and a rank's share at N = 8
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || tail -5 gpurun_out/build.log
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_fullsize.py -m gpu -q -x -k "tbk or c2" 2>&1 | tail -2
for ty in 128 32; do
timeout 300 python bench.py --tile $ty --steps 10 --warmup 3 --no-e2e --no-cpu-baseline > /tmp/b.log 2>&1; tail -1 /tmp/b.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('rows=16384 TY=$ty', round(d['value'],1), round(d['roofline']['frac'],3), round(d['kernel_ms_avg'],4), d['clocks']['sm_mhz'])" || tail -3 /tmp/b.log
done
for ty in 64 32; do
PK_BENCH_ROWS=2048 timeout 300 python bench.py --tile $ty --steps 10 --warmup 3 --no-e2e --no-cpu-baseline > /tmp/b.log 2>&1; tail -1 /tmp/b.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('rows=2048 TY=$ty', round(d['value'],1), round(d['roofline']['frac'],3), round(d['kernel_ms_avg'],4), d['clocks']['sm_mhz'])" || tail -3 /tmp/b.log
done
