# round 2, call 80: heat3d_tb2 planes per block re-swept with the final kernel (ZC 32..128), alternating
run() {
  timeout 300 python bench.py --workload heat3d --steps 10 --no-e2e --no-cpu-baseline --no-e3 $2 > /tmp/b.json 2> /tmp/b.err
  tail -1 /tmp/b.json | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$1', round(d['value'],1), 'frac', round(d['roofline']['frac'],4), 'kms', round(d['kernel_ms_avg'],4), d['clocks']['sm_mhz'])" || tail -3 /tmp/b.err
}
for r in 1 2; do
  for zc in 64 32 48 80 96 128; do run "ZC=$zc" "--tile $zc"; done
done
