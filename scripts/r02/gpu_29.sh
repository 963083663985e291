# round 2, call 29: heat3d_tb2 with sweep-1 boundary rows exchanged between warps through shared
# memory (PK_HEATTB_XCHG=1: 18 instead of 24 sweep-1 rows per block and plane, no spills) vs recompute
run() {
  PK_NVCC_FLAGS="$2" python -m paper_conf_icppw_matzdf20_b200.build > /dev/null 2>&1 || echo BUILD FAIL $2
  timeout 300 python bench.py --workload heat3d --steps 10 --no-e2e --no-cpu-baseline --no-e3 > /tmp/b.json 2> /tmp/b.err
  tail -1 /tmp/b.json | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$1', round(d['value'],1), 'frac', round(d['roofline']['frac'],4), 'kms', round(d['kernel_ms_avg'],4), d['clocks']['sm_mhz'], d['clocks']['reasons'])" || tail -3 /tmp/b.err
}
for r in 1 2 3; do
  run "recompute" "-DPK_HEATTB_XCHG=0"
  run "exchange " "-DPK_HEATTB_XCHG=1"
done
PK_NVCC_FLAGS="-DPK_HEATTB_XCHG=1" python -m paper_conf_icppw_matzdf20_b200.build > /dev/null 2>&1
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_fullsize.py tests/test_gpu_access.py tests/test_gpu_trace.py -q -x -k "heat or c3" > gpurun_out/r02_29_pytest.log 2>&1; echo "exchange parity: $(tail -1 gpurun_out/r02_29_pytest.log)"
mkdir -p gpurun_out/r02_29
timeout 600 ncu --set full --clock-control none --import-source on -k regex:heat3d_tb2 -s 3 -c 1 -o gpurun_out/r02_29/heat_xchg python bench.py --workload heat3d --steps 2 --warmup 3 --no-e2e --no-cpu-baseline --no-e3 > /dev/null 2>&1; echo ncu rc $?
