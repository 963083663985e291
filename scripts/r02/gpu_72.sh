# round 2, call 72: jacobi2d_tb with the fused halo push: GPU suite (push bit-identity, access recording
# incl. the push variant's stores), C1 at P = 2 pulled vs pushed
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r02_72_build.log 2>&1 || tail -5 gpurun_out/r02_72_build.log
timeout 1800 python -m pytest tests -m gpu -q -x > gpurun_out/r02_72_pytest_gpu.log 2>&1; echo "gpu suite: $(tail -1 gpurun_out/r02_72_pytest_gpu.log)"
grep -E "^E |FAILED" gpurun_out/r02_72_pytest_gpu.log | head -6
for r in 1 2 3; do
  for mode in pull push; do
    extra=""; [ $mode = push ] && extra="--push"
    timeout 300 python bench.py --workload jacobi2d --parts 2 --no-e2e --no-cpu-baseline --no-e3 $extra > /tmp/b.json 2> /tmp/e; tail -1 /tmp/b.json | python -c "import json,sys; d=json.loads(sys.stdin.read()); t=d['transfers']; print('C1 tb5 P=2 $mode', round(d['value'],1), 'moved', t['moved_bytes'], 'pushed', t['pushed_bytes'], 'min', t['analytic_min_bytes'])" || tail -3 /tmp/e
  done
done
