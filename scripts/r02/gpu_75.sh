# round 2, call 75: jacobi2d_tb with register row strips (3 shared loads per cell): parity, C1 bench, launch list
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r02_75_build.log 2>&1 || tail -5 gpurun_out/r02_75_build.log
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_trace.py tests/test_gpu_access.py -q -x -k "jacobi" > gpurun_out/r02_75_pytest.log 2>&1; echo "jacobi tests: $(tail -1 gpurun_out/r02_75_pytest.log)"
for r in 1 2 3; do
  timeout 300 python bench.py --workload jacobi2d --no-e2e --no-cpu-baseline > /tmp/b.json 2> /tmp/e; tail -1 /tmp/b.json | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('C1 P=1', round(d['value'],1), 'us/step', round(1e3*d['ms_per_step'],1))" || tail -3 /tmp/e
  timeout 300 python bench.py --workload jacobi2d --parts 2 --no-e2e --no-cpu-baseline --no-e3 > /tmp/b.json 2> /tmp/e; tail -1 /tmp/b.json | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('C1 P=2', round(d['value'],1), 'us/step', round(1e3*d['ms_per_step'],1))" || tail -3 /tmp/e
done
python bench.py --workload jacobi2d --steps 2 --warmup 3 --no-e2e --no-cpu-baseline --no-e3 > gpurun_out/r02_75_plain.log 2>&1 &&
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/r02_75_launches.csv python bench.py --workload jacobi2d --steps 2 --warmup 3 --no-e2e --no-cpu-baseline --no-e3 > /dev/null 2>&1
python scripts/launch_summary.py gpurun_out/r02_75_launches.csv "bench --workload jacobi2d" | head -3
