# round 2, call 34: sustained (power-limited) roofs.  Board power + SM clock while (1) torch D2D
# copies run back to back for 4 s, (2) C2 / C3 benches run ~2.5 s, (3) the same benches at the
# default length; burst copy for reference.
pw() {   # $1 = tag, rest = command
  local tag=$1; shift
  nvidia-smi --query-gpu=power.draw,clocks.sm --format=csv,noheader,nounits -lms 100 > /tmp/pw.csv &
  local SMI=$!
  "$@" > /tmp/out.txt 2> /tmp/err.txt
  kill $SMI
  cp /tmp/pw.csv gpurun_out/r02_34_power_$tag.csv
  python - "$tag" <<'PY'
import sys, json
rows=[l.split(',') for l in open('/tmp/pw.csv') if l.strip()]
pw=[float(r[0]) for r in rows]; mx=max(pw)
clk=sorted(float(r[1]) for r in rows if float(r[0])>0.9*mx)
line=[l for l in open('/tmp/out.txt') if l.startswith('{')][-1]
d=json.loads(line)
if 'd2d_copy_sustained' in d:
    s=d['d2d_copy_sustained']; b=d['d2d_copy_burst']
    v=f"copy sustained {s['gbs_read_plus_write']:.1f} GB/s over {s['seconds']:.2f} s, burst {b['gbs_read_plus_write']:.1f} GB/s"
else:
    v=f"{d['value']:.1f} {d['unit']} frac {d['roofline']['frac']:.4f} ms/step {d['ms_per_step']:.2f} steps {d['steps']} clocks {d['clocks']['sm_mhz']}"
print(sys.argv[1], v, '| W max', mx, 'SM MHz at >90% of max W', clk[len(clk)//2] if clk else None)
PY
}
for r in 1 2; do
  pw copy python scripts/probe_peaks.py --sustained 4
  pw c2_long python bench.py --workload hotspot2d --steps 170 --no-e2e --no-cpu-baseline --no-e3
  pw c3_long python bench.py --workload heat3d --steps 60 --no-e2e --no-cpu-baseline --no-e3
  pw c2_default python bench.py --workload hotspot2d --no-e2e --no-cpu-baseline --no-e3
  pw c3_default python bench.py --workload heat3d --no-e2e --no-cpu-baseline --no-e3
done
