# Re-entry verification: full GPU suite, smoke, every bench line, launch list + ncu of heat3d_tb2
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || true
timeout 1500 python -m pytest tests -m gpu -q > gpurun_out/pytest_gpu.log 2>&1; echo "PYTEST: $(tail -1 gpurun_out/pytest_gpu.log)"
grep -E "FAILED|Error" gpurun_out/pytest_gpu.log | head -5
timeout 300 python -c "import __graft_entry__ as g; g.smoke(); print('SMOKE OK')" > gpurun_out/smoke.log 2>&1; tail -1 gpurun_out/smoke.log
timeout 600 python bench.py > gpurun_out/bench_default.log 2>&1; tail -1 gpurun_out/bench_default.log > gpurun_out/bench_default.json
timeout 300 python bench.py --impl reference --steps 3 --warmup 1 > gpurun_out/bench_reference.log 2>&1; tail -1 gpurun_out/bench_reference.log > gpurun_out/bench_reference.json
for w in heat3d sgemm nbody jacobi2d; do
  timeout 600 python bench.py --workload $w --steps 5 --warmup 3 > gpurun_out/bench_$w.log 2>&1; tail -1 gpurun_out/bench_$w.log > gpurun_out/bench_$w.json
done
for f in gpurun_out/bench_*.json; do python -c "
import json,sys; d=json.load(open('$f')); print('$f', d.get('value'), d.get('unit'), (d.get('roofline') or {}).get('frac'), (d.get('config') or {}).get('kernel'))" 2>&1 | tail -1; done
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/launches_default.csv python bench.py --steps 2 --warmup 1 --no-e2e --no-cpu-baseline > gpurun_out/launches_default.log 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/launches_heat3d.csv python bench.py --workload heat3d --steps 1 --warmup 1 --no-e2e --no-cpu-baseline > gpurun_out/launches_heat3d.log 2>&1
timeout 400 ncu --set full --clock-control none --import-source on -k regex:heat -s 5 -c 1 -o gpurun_out/prof_heat_tb2 python bench.py --workload heat3d --steps 1 --warmup 1 --iters 12 --no-e2e --no-cpu-baseline > gpurun_out/prof_heat_tb2.log 2>&1
ls gpurun_out
