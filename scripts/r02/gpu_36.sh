# round 2, call 36: is the staged path (TMA -> shared -> registers) the power sink?  One-sweep
# kernels, sustained (~3 s) vs default length: TMA-ring vs register-window (LDG/STG only) variants
pw() {   # $1 = tag, rest = command
  local tag=$1; shift
  nvidia-smi --query-gpu=power.draw,clocks.sm --format=csv,noheader,nounits -lms 100 > /tmp/pw.csv &
  local SMI=$!
  "$@" > /tmp/out.txt 2> /tmp/err.txt
  kill $SMI
  python - "$tag" <<'PY'
import sys, json
rows=[l.split(',') for l in open('/tmp/pw.csv') if l.strip()]
pw=[float(r[0]) for r in rows]; mx=max(pw)
clk=sorted(float(r[1]) for r in rows if float(r[0])>0.9*mx)
lines=[l for l in open('/tmp/out.txt') if l.startswith('{')]
if not lines: print(sys.argv[1], 'FAILED', open('/tmp/err.txt').read()[-300:]); sys.exit()
d=json.loads(lines[-1])
v=f"{d['value']:.1f} {d['unit']} frac {d['roofline']['frac']:.4f} steps {d['steps']} kms {d.get('kernel_ms_avg')} clocks {d['clocks']['sm_mhz']}"
print(sys.argv[1], v, '| W max', mx, 'SM MHz at >90% of max W', clk[len(clk)//2] if clk else None)
PY
}
for r in 1 2; do
  pw heat3d_tma_long python bench.py --workload heat3d --variant heat3d --steps 60 --no-e2e --no-cpu-baseline --no-e3
  pw heat3d_regs_long python bench.py --workload heat3d --variant heat3d_regs --steps 60 --no-e2e --no-cpu-baseline --no-e3
  pw hotspot_tma_long python bench.py --workload hotspot2d --variant hotspot2d --steps 100 --no-e2e --no-cpu-baseline --no-e3
  pw hotspot_regs_long python bench.py --workload hotspot2d --variant hotspot2d_regs --steps 100 --no-e2e --no-cpu-baseline --no-e3
done
