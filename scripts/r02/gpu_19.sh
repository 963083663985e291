# round 2, call 19: checkpoint -- racecheck reproducer, smoke, every bench line, reference arm, C2 launch list
nvcc -gencode arch=compute_100a,code=sm_100a -o /tmp/rr scripts/racecheck_bulk_ring.cu -lcuda > /dev/null 2>&1
{ for m in 0 1; do echo "== mode $m"; /tmp/rr $m; compute-sanitizer --tool racecheck /tmp/rr $m 2>&1 | grep -E "RACECHECK SUMMARY|hazard|Race reported" | head -4; done; } > gpurun_out/r02_19_racecheck.txt 2>&1; cat gpurun_out/r02_19_racecheck.txt
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r02_19_build.log 2>&1 || tail -5 gpurun_out/r02_19_build.log
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r02_19_smoke.log 2>&1; tail -1 gpurun_out/r02_19_smoke.log
for w in hotspot2d heat3d sgemm nbody jacobi2d; do
  timeout 900 python bench.py --workload $w > gpurun_out/r02_19_$w.json 2> gpurun_out/r02_19_$w.err
  tail -1 gpurun_out/r02_19_$w.json | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$w', round(d['value'],1), d['unit'], 'frac', round((d.get('roofline') or {}).get('frac',0),4), 'e2e', round((d.get('e2e') or {}).get('value',0),1), 'host', round(d['host_us_per_launch'],2), 'E3', (d.get('e3_single_gpu_slowdown') or {}).get('slowdown_pct'), d['clocks']['sm_mhz'], d['clocks']['reasons'])" || tail -3 gpurun_out/r02_19_$w.err
done
timeout 600 python bench.py --impl reference --steps 3 --warmup 3 > gpurun_out/r02_19_reference.json 2>&1; tail -c 300 gpurun_out/r02_19_reference.json
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/r02_19_launches_c2.csv python bench.py --steps 2 --warmup 3 --no-e2e --no-cpu-baseline --no-e3 > /dev/null 2>&1
python scripts/launch_summary.py gpurun_out/r02_19_launches_c2.csv "python bench.py --steps 2 --warmup 3 --no-e2e --no-cpu-baseline --no-e3" | head -8
