# hotspot2d_tbk with programmatic dependent launch (PK_PDL=1): full C2 and one rank's N = 8 share (2048 rows)
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || tail -5 gpurun_out/build.log
PK_PDL=1 timeout 900 python -m pytest tests -m gpu -x -q -k "hotspot or tbk or graph or spmd" > gpurun_out/pytest_pdl.log 2>&1; echo "PDL tests: $(tail -1 gpurun_out/pytest_pdl.log)"
run() {
  timeout 300 env $1 python bench.py --steps 10 --warmup 3 --no-e2e --no-cpu-baseline > /tmp/b.log 2>&1; tail -1 /tmp/b.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$1', round(d['value'],1), round(d['roofline']['frac'],3), round(d['kernel_ms_avg'],4), round(d['ms_per_step'],3), d['clocks']['sm_mhz'], d['config'].get('rows_per_tile'))" || tail -3 /tmp/b.log
}
for r in 1 2; do
run PK_PDL=0; run PK_PDL=1; run "PK_PDL=0 PK_BENCH_ROWS=2048"; run "PK_PDL=1 PK_BENCH_ROWS=2048"
done
