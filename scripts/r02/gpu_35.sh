# round 2, call 35: consumer mbarrier waits with a suspend-time hint (PK_MBAR_HINT_NS) -- does
# less polling lower the board power of the sustained (power-capped) C2 / C3 runs?
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
line=[l for l in open('/tmp/out.txt') if l.startswith('{')][-1]
d=json.loads(line)
v=f"{d['value']:.1f} {d['unit']} frac {d['roofline']['frac']:.4f} steps {d['steps']} clocks {d['clocks']['sm_mhz']}"
print(sys.argv[1], v, '| W max', mx, 'SM MHz at >90% of max W', clk[len(clk)//2] if clk else None)
PY
}
for r in 1 2; do
  for h in 0 2000 100000; do
    PK_NVCC_FLAGS="-DPK_MBAR_HINT_NS=$h" python -m paper_conf_icppw_matzdf20_b200.build > /dev/null 2>&1 || echo BUILD FAIL
    pw "hint$h c2_long" python bench.py --workload hotspot2d --steps 170 --no-e2e --no-cpu-baseline --no-e3
    pw "hint$h c3_long" python bench.py --workload heat3d --steps 60 --no-e2e --no-cpu-baseline --no-e3
    pw "hint$h c2_short" python bench.py --workload hotspot2d --no-e2e --no-cpu-baseline --no-e3
  done
done
