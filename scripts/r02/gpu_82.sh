# round 2, call 82: end-of-session check of the committed state -- build, GPU suite, smoke, default bench
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r02_82_build.log 2>&1 || tail -5 gpurun_out/r02_82_build.log
timeout 1800 python -m pytest tests -m gpu -q > gpurun_out/r02_82_pytest_gpu.log 2>&1; echo "gpu suite: $(tail -1 gpurun_out/r02_82_pytest_gpu.log)"
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r02_82_smoke.log 2>&1; tail -1 gpurun_out/r02_82_smoke.log
timeout 600 python bench.py > gpurun_out/r02_82_bench.json 2> gpurun_out/r02_82_bench.err; tail -1 gpurun_out/r02_82_bench.json | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('bench', round(d['value'],1), d['unit'], 'frac', round(d['roofline']['frac'],4), 'e2e', round(d['e2e']['value'],1), 'cpu', round(d['cpu_baseline']['value'],2), d['clocks'])"
