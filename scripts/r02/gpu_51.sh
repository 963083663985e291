# round 2, call 51: cost of heat3d_tb2's clamping (EDGE) consumer: every block through it vs as built
run() {
  PK_NVCC_FLAGS="$2" python -m paper_conf_icppw_matzdf20_b200.build > /dev/null 2>&1 || echo BUILD FAIL $2
  timeout 300 python bench.py --workload heat3d --steps 10 --no-e2e --no-cpu-baseline --no-e3 > /tmp/b.json 2> /tmp/b.err
  tail -1 /tmp/b.json | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$1', round(d['value'],1), 'frac', round(d['roofline']['frac'],4), 'kms', round(d['kernel_ms_avg'],4), d['clocks']['sm_mhz'], d['clocks']['reasons'])" || tail -3 /tmp/b.err
}
for r in 1 2 3; do
  run "as built " ""
  run "all edge " "-DPK_HEATTB_ALLEDGE"
done
python -m paper_conf_icppw_matzdf20_b200.build > /dev/null 2>&1
