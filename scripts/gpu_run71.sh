# Checkpoint: full GPU suite, smoke, every bench line (live kernel events, pipelined e2e), reference arm, launch lists
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || true
timeout 1500 python -m pytest tests -m gpu -q > gpurun_out/pytest_gpu.log 2>&1; echo "PYTEST: $(tail -1 gpurun_out/pytest_gpu.log)"
grep -E "FAILED|Error" gpurun_out/pytest_gpu.log | head -5
timeout 300 python -c "import __graft_entry__ as g; g.smoke(); print('SMOKE OK')" > gpurun_out/smoke.log 2>&1; tail -1 gpurun_out/smoke.log
timeout 900 python bench.py > gpurun_out/bench_default.log 2>gpurun_out/bench_default.err; tail -1 gpurun_out/bench_default.log > gpurun_out/bench_default.json; tail -1 gpurun_out/bench_default.err
timeout 300 python bench.py --impl reference --steps 3 --warmup 1 > gpurun_out/bench_reference.log 2>&1; tail -1 gpurun_out/bench_reference.log > gpurun_out/bench_reference.json
for w in heat3d sgemm nbody jacobi2d; do
  timeout 900 python bench.py --workload $w --steps 5 --warmup 3 > gpurun_out/bench_$w.log 2>&1; tail -1 gpurun_out/bench_$w.log > gpurun_out/bench_$w.json
done
timeout 600 python bench.py --workload jacobi2d --parts 2 --steps 5 --warmup 3 > gpurun_out/bench_jacobi_p2.log 2>&1; tail -1 gpurun_out/bench_jacobi_p2.log > gpurun_out/bench_jacobi_p2.json
for f in gpurun_out/bench_*.json; do python -c "
import json; d=json.load(open('$f')); print('$f', d.get('value'), d.get('unit'), (d.get('roofline') or {}).get('frac'), (d.get('e2e') or {}).get('value'), (d.get('clocks') or {}).get('reasons'))" 2>&1 | tail -1; done
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/launches_default.csv python bench.py --steps 2 --warmup 1 --no-e2e --no-cpu-baseline > gpurun_out/launches_default.log 2>&1
