# round 2, call 48: push as a post-pass of the pushed rows (tbk per tile, heat tb2 per plane): GPU suite, then push vs pull at
# P = 2/8 virtual partitions (C2, C3) as in call 45
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r02_48_build.log 2>&1 || tail -5 gpurun_out/r02_48_build.log
timeout 1800 python -m pytest tests -m gpu -q -x > gpurun_out/r02_48_pytest_gpu.log 2>&1; echo "gpu suite: $(tail -1 gpurun_out/r02_48_pytest_gpu.log)"
: > gpurun_out/r02_48_push.txt
for rep in 1 2; do
  for spec in "hotspot2d 2" "hotspot2d 8" "heat3d 2" "heat3d 8" "jacobi2d 2"; do
    set -- $spec; w=$1; P=$2
    for mode in pull push; do
      extra=""; [ $mode = push ] && extra="--push"
      timeout 600 python bench.py --workload $w --parts $P --steps 10 --warmup 3 --no-e2e --no-cpu-baseline --no-e3 $extra > /tmp/b.log 2>&1
      tail -1 /tmp/b.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); t=d['transfers']; print('$mode $w P=$P', round(d['value'],2), d['unit'], 'ms/step', round(d['ms_per_step'],4), 'moved', t['moved_bytes'], 'pushed', t['pushed_bytes'], 'min', t['analytic_min_bytes'], d['clocks']['sm_mhz'])" >> gpurun_out/r02_48_push.txt 2>&1 || tail -3 /tmp/b.log >> gpurun_out/r02_48_push.txt
    done
  done
done
cat gpurun_out/r02_48_push.txt
