python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || tail -5 gpurun_out/build.log
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_fullsize.py tests/test_gpu_spmd_ipc.py -m gpu -q -x -k "heat" 2>&1 | tail -1
timeout 600 python bench.py --workload heat3d --steps 5 --warmup 3 > gpurun_out/bench_heat3d.log 2>&1; tail -1 gpurun_out/bench_heat3d.log > gpurun_out/bench_heat3d.json
python -c "import json; d=json.load(open('gpurun_out/bench_heat3d.json')); print(d['value'], d['roofline']['frac'], d['e2e']['value'], d['clocks'])"
timeout 400 ncu --set full --clock-control none --import-source on -k regex:heat -s 5 -c 1 -o gpurun_out/prof_heat_tb2_nw4 python bench.py --workload heat3d --steps 1 --warmup 1 --iters 12 --no-e2e --no-cpu-baseline > gpurun_out/prof_heat_tb2_nw4.log 2>&1
