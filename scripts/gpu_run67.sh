# async host copies: GPU tests, then full bench lines (default + heat3d) with the pipelined e2e
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || tail -5 gpurun_out/build.log
timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -q -x -k "async or graph or push_hotspot_tbk" 2>&1 | tail -2
timeout 600 python bench.py > gpurun_out/bench_default.log 2>&1; tail -1 gpurun_out/bench_default.log > gpurun_out/bench_default.json
python -c "import json; d=json.load(open('gpurun_out/bench_default.json')); print(d['value'], d['roofline'], d['e2e'], d['kernel_timing'])" || tail -5 gpurun_out/bench_default.log
