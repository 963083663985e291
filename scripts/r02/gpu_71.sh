# round 2, call 71: C1 bench default now jacobi2d_tb (K = 5, two launches per 10-sweep step): GPU suite,
# default C1 line at P = 1 and P = 2, the one-sweep kernel beside it
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r02_71_build.log 2>&1 || tail -5 gpurun_out/r02_71_build.log
timeout 1800 python -m pytest tests -m gpu -q -x > gpurun_out/r02_71_pytest_gpu.log 2>&1; echo "gpu suite: $(tail -1 gpurun_out/r02_71_pytest_gpu.log)"
for r in 1 2; do
  timeout 300 python bench.py --workload jacobi2d > gpurun_out/r02_71_c1_$r.json 2> /tmp/e; tail -1 gpurun_out/r02_71_c1_$r.json | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('C1 default', d['config']['kernel'], d['config']['sweeps_per_launch'], round(d['value'],1), 'e2e', round(d['e2e']['value'],1), 'E3', d['e3_single_gpu_slowdown']['slowdown_pct'], 'launches', d['gpu_launches'])" || tail -3 /tmp/e
  timeout 300 python bench.py --workload jacobi2d --parts 2 --no-e2e --no-cpu-baseline --no-e3 > /tmp/b.json 2> /tmp/e; tail -1 /tmp/b.json | python -c "import json,sys; d=json.loads(sys.stdin.read()); t=d['transfers']; print('C1 default P=2', round(d['value'],1), 'moved', t['moved_bytes'], 'min', t['analytic_min_bytes'])" || tail -3 /tmp/e
  timeout 300 python bench.py --workload jacobi2d --variant jacobi2d --no-e2e --no-cpu-baseline --no-e3 > /tmp/b.json 2> /tmp/e; tail -1 /tmp/b.json | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('C1 one-sweep', round(d['value'],1))" || tail -3 /tmp/e
done
