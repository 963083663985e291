# round 2, call 58: GPU suite with heat3d_tb3 (parity, remainder sweeps, push, access recording, poison),
# then the C3 bench line with --variant heat3d_tb3 at the config's 50 sweeps
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r02_58_build.log 2>&1 || tail -5 gpurun_out/r02_58_build.log
timeout 1800 python -m pytest tests -m gpu -q -x > gpurun_out/r02_58_pytest_gpu.log 2>&1; echo "gpu suite: $(tail -1 gpurun_out/r02_58_pytest_gpu.log)"
grep -E "^E |FAILED" gpurun_out/r02_58_pytest_gpu.log | head -8
timeout 300 python bench.py --workload heat3d --variant heat3d_tb3 --no-cpu-baseline > gpurun_out/r02_58_tb3.json 2> gpurun_out/r02_58_tb3.err; tail -1 gpurun_out/r02_58_tb3.json | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('tb3 variant', round(d['value'],1), d['unit'], 'frac', round(d['roofline']['frac'],4), 'e2e', round(d['e2e']['value'],1), 'launches', d['gpu_launches'], d['clocks'])" || tail -3 gpurun_out/r02_58_tb3.err
