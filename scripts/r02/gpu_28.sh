# round 2, call 28: heat3d_tb2 producer back-off (PK_HEATTB_PNS) and ring depth (PK_HEATTB_NS)
run() {
  PK_NVCC_FLAGS="$2" python -m paper_conf_icppw_matzdf20_b200.build > /dev/null 2>&1 || echo BUILD FAIL $2
  timeout 300 python bench.py --workload heat3d --steps 8 --no-e2e --no-cpu-baseline --no-e3 > /tmp/b.json 2> /tmp/b.err
  tail -1 /tmp/b.json | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$1', round(d['value'],1), 'frac', round(d['roofline']['frac'],4), d['clocks']['sm_mhz'], d['clocks']['reasons'])" || tail -3 /tmp/b.err
}
for r in 1 2; do
run "PNS256 NS6" "-DPK_HEATTB_PNS=256"
run "PNS64 NS6" "-DPK_HEATTB_PNS=64"
run "PNS128 NS6" "-DPK_HEATTB_PNS=128"
run "PNS512 NS6" "-DPK_HEATTB_PNS=512"
run "PNS256 NS5" "-DPK_HEATTB_PNS=256 -DPK_HEATTB_NS=5"
done
