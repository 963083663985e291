# round 2, call 30: heat3d_tb2 exchange variant: interior-column blocks without x-clamp selects
# (PK_HEATTB_CEDGE=1, no spills now) and ring depth 5, against recompute / exchange
run() {
  PK_NVCC_FLAGS="$2" python -m paper_conf_icppw_matzdf20_b200.build > /dev/null 2>&1 || echo BUILD FAIL $2
  timeout 300 python bench.py --workload heat3d --steps 10 --no-e2e --no-cpu-baseline --no-e3 > /tmp/b.json 2> /tmp/b.err
  tail -1 /tmp/b.json | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$1', round(d['value'],1), 'frac', round(d['roofline']['frac'],4), 'kms', round(d['kernel_ms_avg'],4), d['clocks']['sm_mhz'], d['clocks']['reasons'])" || tail -3 /tmp/b.err
}
for r in 1 2 3; do
  run "recompute     " "-DPK_HEATTB_XCHG=0"
  run "exchange      " "-DPK_HEATTB_XCHG=1"
  run "exchange cedge" "-DPK_HEATTB_XCHG=1 -DPK_HEATTB_CEDGE=1"
  run "exchange ns5  " "-DPK_HEATTB_XCHG=1 -DPK_HEATTB_NS=5"
done
PK_NVCC_FLAGS="-DPK_HEATTB_XCHG=1 -DPK_HEATTB_CEDGE=1" python -m paper_conf_icppw_matzdf20_b200.build > /dev/null 2>&1
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_fullsize.py -q -x -k "heat or c3" > gpurun_out/r02_30_pytest.log 2>&1; echo "cedge parity: $(tail -1 gpurun_out/r02_30_pytest.log)"
