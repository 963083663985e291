# round 2, call 56: heat3d_tb3 pipeline waits with a suspend-time hint (0 = spin / 200 / 1000 / 5000 ns)
# and the sweep-1 ring depth, vs tb2 in alternation
run() {
  PK_NVCC_FLAGS="$3" python -m paper_conf_icppw_matzdf20_b200.build > /dev/null 2>&1 || echo BUILD FAIL $3
  timeout 300 python bench.py --workload heat3d --iters 48 --steps 10 --no-e2e --no-cpu-baseline --no-e3 $2 > /tmp/b.json 2> /tmp/b.err
  tail -1 /tmp/b.json | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$1', round(d['value'],1), 'frac', round(d['roofline']['frac'],4), 'kms', round(d['kernel_ms_avg'],4), d['clocks']['sm_mhz'], d['clocks']['reasons'], d['clocks'].get('power_w_max'))" || tail -3 /tmp/b.err
}
T="--variant heat3d_tb3 --tile 64"
for r in 1 2; do
  run "tb2            " "" ""
  run "tb3 spin       " "$T" ""
  run "tb3 hint200    " "$T" "-DPK_HEATTB3_HINT=200"
  run "tb3 hint1000   " "$T" "-DPK_HEATTB3_HINT=1000"
  run "tb3 hint5000   " "$T" "-DPK_HEATTB3_HINT=5000"
  run "tb3 nl1=4 ns=5 " "$T" "-DPK_HEATTB3_NL1=4 -DPK_HEATTB3_NS=5"
done
python -m paper_conf_icppw_matzdf20_b200.build > /dev/null 2>&1
