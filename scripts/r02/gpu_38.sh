# round 2, call 38: pk_launch_sequence (one graph per launch sequence): GPU tests, C1 bench line
# (10 sweeps per step as one sequence) and the other workloads unchanged
python -m paper_conf_icppw_matzdf20_b200.build > /dev/null 2>&1 || echo BUILD FAIL
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "sequence or c1 or jacobi or graph or capture" > gpurun_out/r02_38_pytest.log 2>&1; echo "parity: $(tail -1 gpurun_out/r02_38_pytest.log)"
for r in 1 2; do
  timeout 600 python bench.py --workload jacobi2d > gpurun_out/r02_38_jacobi2d.json 2> gpurun_out/r02_38_jacobi2d.err
  tail -1 gpurun_out/r02_38_jacobi2d.json | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('jacobi2d', round(d['value'],1), d['unit'], 'frac', round((d.get('roofline') or {}).get('frac',0),4), 'kms', d.get('kernel_ms_avg'), 'ms/step', round(d['ms_per_step'],4), 'e2e', round((d.get('e2e') or {}).get('value',0),1), 'host', round(d['host_us_per_launch'],2), 'E3', (d.get('e3_single_gpu_slowdown') or {}).get('slowdown_pct'), 'launches', d.get('gpu_launches'))" || tail -3 gpurun_out/r02_38_jacobi2d.err
  timeout 600 python bench.py --workload jacobi2d --parts 2 --no-e2e --no-cpu-baseline > /tmp/j2.json 2> /tmp/j2.err
  tail -1 /tmp/j2.json | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('jacobi2d P=2', round(d['value'],1), 'ms/step', round(d['ms_per_step'],4), d['transfers'])" || tail -3 /tmp/j2.err
done
