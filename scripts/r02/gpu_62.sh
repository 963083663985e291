# round 2, call 62: C1 (latency-bound) bench A/B: current build vs the build from the start of this
# session (scratch/libpk_before_passes.so), alternating, to separate a regression from box variance
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
for r in 1 2 3; do
  for lib in new old; do
    if [ $lib = old ]; then export PK_LIB_OVERRIDE=$PWD/scratch/libpk_before_passes.so; else unset PK_LIB_OVERRIDE; fi
    timeout 300 python bench.py --workload jacobi2d --no-e2e --no-cpu-baseline > /tmp/b.json 2> /tmp/b.err
    tail -1 /tmp/b.json | python -c "import json,sys; d=json.loads(sys.stdin.read()); e=d['e3_single_gpu_slowdown']; print('$lib', round(d['value'],1), 'ms/step', round(d['ms_per_step'],4), 'host', round(d['host_us_per_launch'],2), 'lib/direct ms', round(e['library_ms_per_step'],4), round(e['direct_ms_per_step'],4))" || tail -3 /tmp/b.err
  done
done
unset PK_LIB_OVERRIDE
