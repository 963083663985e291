# end of round 1: GPU suite, smoke, and one bench line per workload with the final kernels
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || tail -5 gpurun_out/build.log
timeout 900 python -m pytest tests -m gpu -q > gpurun_out/pytest_gpu_final.log 2>&1; echo "gpu suite: $(tail -1 gpurun_out/pytest_gpu_final.log)"
python -c "import __graft_entry__ as g; g.smoke(); print('smoke ok')" > gpurun_out/smoke_final.log 2>&1; tail -1 gpurun_out/smoke_final.log
for w in hotspot2d heat3d sgemm nbody jacobi2d; do
  timeout 600 python bench.py --workload $w > gpurun_out/final_$w.json 2> gpurun_out/final_$w.err
  tail -1 gpurun_out/final_$w.json | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$w', round(d['value'],1), d['unit'], (d.get('roofline') or {}).get('frac'), (d.get('e2e') or {}).get('value'), d['clocks']['sm_mhz'], d['clocks']['reasons'])" || tail -3 gpurun_out/final_$w.err
done
timeout 600 python bench.py --impl reference --steps 3 --warmup 3 > gpurun_out/final_reference.json 2>&1; tail -c 300 gpurun_out/final_reference.json
