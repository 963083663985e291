# round 2, call 32: heat3d_tb2 with sweep 1's z-minus rows kept in registers (PK_HEATTB_ZREG=1:
# 8 instead of 12 shared loads per warp and plane for the own rows) -- less energy per update?
run() {
  PK_NVCC_FLAGS="$2" python -m paper_conf_icppw_matzdf20_b200.build > /dev/null 2>&1 || echo BUILD FAIL $2
  nvidia-smi --query-gpu=power.draw,clocks.sm --format=csv,noheader,nounits -lms 100 > /tmp/pw.csv &
  SMI=$!
  timeout 300 python bench.py --workload heat3d --steps 30 --no-e2e --no-cpu-baseline --no-e3 > /tmp/b.json 2> /tmp/b.err
  kill $SMI
  PW=$(python -c "
rows=[l.split(',') for l in open('/tmp/pw.csv') if l.strip()]
pw=sorted(float(r[0]) for r in rows if float(r[0])>700)
print('W>700:', len(pw), 'median', pw[len(pw)//2] if pw else None)")
  tail -1 /tmp/b.json | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$1', round(d['value'],1), 'frac', round(d['roofline']['frac'],4), 'kms', round(d['kernel_ms_avg'],4), d['clocks']['sm_mhz'], d['clocks']['reasons'], '$PW')" || tail -3 /tmp/b.err
}
for r in 1 2 3; do
  run "smem zm" "-DPK_HEATTB_ZREG=0"
  run "reg  zm" "-DPK_HEATTB_ZREG=1"
done
PK_NVCC_FLAGS="-DPK_HEATTB_ZREG=1" python -m paper_conf_icppw_matzdf20_b200.build > /dev/null 2>&1
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_fullsize.py -q -x -k "heat or c3" > gpurun_out/r02_32_pytest.log 2>&1; echo "zreg parity: $(tail -1 gpurun_out/r02_32_pytest.log)"
