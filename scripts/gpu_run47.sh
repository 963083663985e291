python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || true
timeout 1200 python -m pytest tests -m gpu -q -x 2>&1 | tail -2
r() { timeout 600 python bench.py $1 --steps 10 --warmup 3 --no-e2e --no-cpu-baseline > /tmp/b.log 2>&1; tail -1 /tmp/b.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$1', round(d['value'],1), round(d['roofline']['frac'],3), round(d['kernel_ms_avg'],4))"; }
for ty in 104 112 116 120 124 128 136; do r "--tile $ty"; done
r "--tile 120"; r "--tile 128"
