# hotspot2d_tbk K = 4: rows per tile (wave quantisation of the persistent grid)
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || tail -5 gpurun_out/build.log
for ty in 128 144 216 264 328 128 216; do
timeout 300 python bench.py --tile $ty --steps 10 --warmup 3 --no-e2e --no-cpu-baseline > /tmp/b.log 2>&1; tail -1 /tmp/b.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('TY=$ty', round(d['value'],1), round(d['roofline']['frac'],3), round(d['kernel_ms_avg'],4), d['clocks']['sm_mhz'])" || tail -3 /tmp/b.log
done
