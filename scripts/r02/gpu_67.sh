# round 2, call 69: jacobi2d_tb templated on K (unrolled, 512 threads): parity, C1 bench lines
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r02_69_build.log 2>&1 || tail -5 gpurun_out/r02_69_build.log
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "jacobi" > gpurun_out/r02_69_pytest.log 2>&1; echo "jacobi parity: $(tail -1 gpurun_out/r02_69_pytest.log)"
run() {
  timeout 300 python bench.py --workload jacobi2d --no-e2e --no-cpu-baseline $2 > /tmp/b.json 2> /tmp/b.err
  tail -1 /tmp/b.json | python -c "import json,sys; d=json.loads(sys.stdin.read()); t=d['transfers']; e=d.get('e3_single_gpu_slowdown') or {}; print('$1', round(d['value'],1), 'ms/step', round(d['ms_per_step'],4), 'launches', d['gpu_launches'], 'moved', t['moved_bytes'], 'E3', e.get('slowdown_pct'))" || tail -3 /tmp/b.err
}
for r in 1 2; do
  run "jacobi2d      P=1" ""
  run "jacobi2d_tb10 P=1" "--variant jacobi2d_tb"
  run "jacobi2d_tb5  P=1" "--variant jacobi2d_tb --sweeps 5"
  run "jacobi2d push P=2" "--parts 2 --no-e3 --push"
  run "jacobi2d_tb10 P=2" "--parts 2 --no-e3 --variant jacobi2d_tb"
  run "jacobi2d_tb5  P=2" "--parts 2 --no-e3 --variant jacobi2d_tb --sweeps 5"
done
