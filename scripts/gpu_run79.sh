python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || tail -5 gpurun_out/build.log
timeout 1200 python -m pytest tests/test_gpu_parity.py tests/test_gpu_fullsize.py tests/test_gpu_spmd_ipc.py -m gpu -q -x -k "nbody" 2>&1 | tail -1
timeout 900 python bench.py --workload nbody --steps 3 --warmup 3 > gpurun_out/bench_nbody.log 2>&1; tail -1 gpurun_out/bench_nbody.log > gpurun_out/bench_nbody.json
python -c "import json; d=json.load(open('gpurun_out/bench_nbody.json')); print(d['value'], d['roofline']['frac'], d['e2e']['value'], d['clocks'])"
timeout 900 ncu --set full --clock-control none --import-source on -k regex:nbody_partial -s 3 -c 1 -o gpurun_out/prof_nbody5 python bench.py --workload nbody --steps 1 --warmup 3 --iters 1 --no-e2e --no-cpu-baseline > gpurun_out/prof_nbody5.log 2>&1
