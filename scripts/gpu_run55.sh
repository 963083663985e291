python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || true
timeout 300 python scripts/tbk_probe.py 2>&1 | tail -12
for k in 4 6 8; do
timeout 300 python bench.py --sweeps $k --iters 96 --steps 5 --warmup 3 --no-e2e --no-cpu-baseline > /tmp/b.log 2>&1; tail -1 /tmp/b.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('K=$k', round(d['value'],1), round(d['roofline']['frac'],3), round(d['kernel_ms_avg'],4), d['clocks'])" || tail -3 /tmp/b.log
done
