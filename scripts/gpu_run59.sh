# heat3d_tb2 v2: 2-slot sweep-1 window interleaved with sweep 2, COLEDGE template, 8-slot ring; ZC sweep
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || tail -5 gpurun_out/build.log
timeout 600 python -m pytest tests/test_gpu_parity.py -m gpu -q -x -k "heat3d_tb2 or heat_tile" 2>&1 | tail -3
for zc in 128 342 64 256 128; do
timeout 300 python bench.py --workload heat3d --tile $zc --steps 5 --warmup 3 --no-e2e --no-cpu-baseline > /tmp/b.log 2>&1; tail -1 /tmp/b.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('ZC=$zc', round(d['value'],1), round(d['roofline']['frac'],3), round(d['kernel_ms_avg'],4), d['clocks']['sm_mhz'], d['clocks']['reasons'])" || tail -3 /tmp/b.log
done
timeout 400 ncu --set full --clock-control none --import-source on -k regex:heat -s 5 -c 1 -o gpurun_out/prof_heat_tb2v2 python bench.py --workload heat3d --steps 1 --warmup 1 --iters 12 --no-e2e --no-cpu-baseline > gpurun_out/prof_heat_tb2v2.log 2>&1
