# round 2, call 31: racecheck / synccheck of heat3d_tb2's exchange buffer; board power during the
# C3 and C2 benches (is the power cap the limit?)
for tool in racecheck synccheck; do
  timeout 600 compute-sanitizer --tool $tool --error-exitcode 9 python scripts/sanitize_heat_tb2.py > gpurun_out/r02_31_$tool.log 2>&1; echo "$tool rc=$?"; tail -3 gpurun_out/r02_31_$tool.log
done
for wl in heat3d hotspot2d sgemm; do
  nvidia-smi --query-gpu=timestamp,power.draw,power.limit,enforced.power.limit,clocks.sm,clocks.mem,temperature.gpu,clocks_throttle_reasons.active --format=csv,noheader -lms 100 > gpurun_out/r02_31_power_$wl.csv &
  SMI=$!
  timeout 300 python bench.py --workload $wl --steps 30 --no-e2e --no-cpu-baseline --no-e3 > /tmp/b.json 2> /tmp/b.err
  kill $SMI
  tail -1 /tmp/b.json | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$wl', round(d['value'],1), 'frac', round(d['roofline']['frac'],4), d['clocks'])"
  python - <<PY
import statistics as st
rows=[l.strip().split(', ') for l in open('gpurun_out/r02_31_power_$wl.csv') if l.strip()]
pw=[float(r[1].split()[0]) for r in rows if r[1].split()[0].replace('.','',1).isdigit()]
lim=rows[0][2]
hi=[p for p in pw if p>300]
print('$wl power samples', len(pw), 'limit', lim, 'median under load', st.median(hi) if hi else None, 'max', max(pw))
PY
done
