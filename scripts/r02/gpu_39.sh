# round 2, call 39: C1 with programmatic dependent launch (griddepcontrol) between sweeps vs without
python -m paper_conf_icppw_matzdf20_b200.build > /dev/null 2>&1 || echo BUILD FAIL
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_access.py tests/test_gpu_trace.py tests/test_gpu_fullsize.py -q -x -k "sequence or c1 or jacobi or graph or capture or push" > gpurun_out/r02_39_pytest.log 2>&1; echo "parity: $(tail -1 gpurun_out/r02_39_pytest.log)"
run() {
  env $2 timeout 600 python bench.py --workload jacobi2d $3 > /tmp/j.json 2> /tmp/j.err
  tail -1 /tmp/j.json | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$1', round(d['value'],1), d['unit'], 'kms', d.get('kernel_ms_avg'), 'ms/step', round(d['ms_per_step'],4), 'e2e', round((d.get('e2e') or {}).get('value',0),1), 'E3', (d.get('e3_single_gpu_slowdown') or {}).get('slowdown_pct'))" || tail -3 /tmp/j.err
}
for r in 1 2 3; do
  run "P=1 pdl   " "PK_X=1" "--no-e2e --no-cpu-baseline"
  run "P=1 no-pdl" "PK_NO_PDL=1" "--no-e2e --no-cpu-baseline"
  run "P=2 pdl   " "PK_X=1" "--parts 2 --no-e2e --no-cpu-baseline"
  run "P=2 no-pdl" "PK_NO_PDL=1" "--parts 2 --no-e2e --no-cpu-baseline"
done
