# graph replay at P = 1: full GPU suite, C1 (P = 1, 2) and C2 bench lines
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || tail -5 gpurun_out/build.log
timeout 1500 python -m pytest tests -m gpu -q -x > gpurun_out/pytest_gpu.log 2>&1; echo "PYTEST: $(tail -1 gpurun_out/pytest_gpu.log)"
grep -E "FAILED|Error" gpurun_out/pytest_gpu.log | head -5
for a in "--workload jacobi2d" "--workload jacobi2d --parts 2" "" "--workload heat3d"; do
timeout 300 python bench.py $a --steps 10 --warmup 3 --no-e2e --no-cpu-baseline > /tmp/b.log 2>&1; tail -1 /tmp/b.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$a', round(d['value'],1), round(d['roofline']['frac'],3), round(d['kernel_ms_avg'],4), d.get('graph_replays'), d.get('host_us_per_launch'), d.get('us_per_launch'))" || tail -3 /tmp/b.log
done
