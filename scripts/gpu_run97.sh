# C1 at P = 2 and C2 at P = 8 (virtual): pull (default) vs fused halo push
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || tail -5 gpurun_out/build.log
for a in "--workload jacobi2d --parts 2" "--workload jacobi2d --parts 2 --push" "--parts 8" "--parts 8 --push" "--workload heat3d --parts 4" "--workload heat3d --parts 4 --push"; do
timeout 300 python bench.py $a --steps 5 --warmup 3 --no-e2e --no-cpu-baseline > /tmp/b.log 2>&1; tail -1 /tmp/b.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); t=d['transfers']; print('$a', round(d['value'],1), 'moved', t['moved_bytes'], 'pushed', t['pushed_bytes'], 'host_us', round(d['host_us_per_launch'],2))" || tail -3 /tmp/b.log
done
