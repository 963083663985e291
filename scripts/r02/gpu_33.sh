# round 2, call 33: where does C3's power go?  Board power and SM clock over ~2-3 s runs of
# heat3d_tb2 as built, heat3d_tb2 with the arithmetic removed (PK_HEATTB_DIAG: same TMA ring,
# loads and stores, the update returns the centre value), and hotspot2d_tbk
run() {
  PK_NVCC_FLAGS="$3" python -m paper_conf_icppw_matzdf20_b200.build > /dev/null 2>&1 || echo BUILD FAIL $3
  nvidia-smi --query-gpu=power.draw,clocks.sm --format=csv,noheader,nounits -lms 100 > /tmp/pw.csv &
  SMI=$!
  timeout 300 python bench.py --workload $2 --steps $4 --no-e2e --no-cpu-baseline --no-e3 > /tmp/b.json 2> /tmp/b.err
  kill $SMI
  cp /tmp/pw.csv gpurun_out/r02_33_power_$1.csv
  PW=$(python -c "
rows=[l.split(',') for l in open('/tmp/pw.csv') if l.strip()]
pw=[float(r[0]) for r in rows]; mx=max(pw)
top=sorted(pw)[-8:]
clk=[float(r[1]) for r in rows if float(r[0])>0.9*mx]
print('W max', mx, 'top8 median', top[4], 'SM MHz at >90% of max W', sorted(clk)[len(clk)//2] if clk else None)")
  tail -1 /tmp/b.json | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$1', round(d['value'],1), 'frac', round(d['roofline']['frac'],4), 'kms', round(d['kernel_ms_avg'],4), 'ms/step', round(d['ms_per_step'],2), d['clocks']['sm_mhz'], d['clocks']['reasons'], '$PW')" || tail -3 /tmp/b.err
}
for r in 1 2; do
  run heat_full heat3d "" 60
  run heat_diag heat3d "-DPK_HEATTB_DIAG" 60
  run hotspot hotspot2d "" 150
done
