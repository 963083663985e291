python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || true
timeout 1200 python -m pytest tests/test_gpu_fullsize.py -m gpu -q -x -k "c3" 2>&1 | tail -3
timeout 600 python bench.py --workload heat3d --steps 5 --warmup 3 > gpurun_out/bench_heat3d.log 2>&1; tail -1 gpurun_out/bench_heat3d.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(d['value'], d['roofline'], d['kernel_ms_avg'])"
ncu --set full --import-source on --clock-control none -k regex:k_heat3d_tb2 -c 1 -s 3 -o gpurun_out/heat_tb2 python bench.py --workload heat3d --no-e2e --no-cpu-baseline --steps 1 --warmup 3 > /dev/null 2>&1
ls gpurun_out | head
