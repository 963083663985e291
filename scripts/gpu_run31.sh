python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || true
timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -q -x -k "tbk" 2>&1 | tail -15
for K in 2 3 4; do
timeout 300 python bench.py --no-e2e --no-cpu-baseline --steps 10 --warmup 3 --variant hotspot2d_tbk --sweeps $K > gpurun_out/b.log 2>&1; tail -1 gpurun_out/b.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('K=$K', d['value'], d['roofline']['frac'], d['kernel_ms_avg'])" || tail -5 gpurun_out/b.log
done
