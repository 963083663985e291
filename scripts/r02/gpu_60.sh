# round 2, call 60: hotspot2d_tbk warps beyond the grid's last column only pace the ring
# (PK_TBK_IDLE_SKIP): hotspot parity (incl. full size), then C2 bench alternating with the old build
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r02_60_build.log 2>&1 || tail -5 gpurun_out/r02_60_build.log
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_fullsize.py -q -x -k "hotspot" > gpurun_out/r02_60_pytest.log 2>&1; echo "hotspot parity: $(tail -1 gpurun_out/r02_60_pytest.log)"
run() {
  PK_NVCC_FLAGS="$2" python -m paper_conf_icppw_matzdf20_b200.build > /dev/null 2>&1 || echo BUILD FAIL $2
  timeout 300 python bench.py --steps 20 --no-e2e --no-cpu-baseline --no-e3 > /tmp/b.json 2> /tmp/b.err
  tail -1 /tmp/b.json | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$1', round(d['value'],1), 'frac', round(d['roofline']['frac'],4), 'kms', round(d['kernel_ms_avg'],4), d['clocks']['sm_mhz'], d['clocks']['reasons'])" || tail -3 /tmp/b.err
}
for r in 1 2 3; do
  run "skip   " ""
  run "noskip " "-DPK_TBK_IDLE_SKIP=0"
done
python -m paper_conf_icppw_matzdf20_b200.build > /dev/null 2>&1
