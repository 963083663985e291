# round 2, call 15: launch list of the sgemm bench (v3) -- where do the per-step gaps come from?
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/r02_15_launches.csv python bench.py --workload sgemm --steps 3 --warmup 3 --no-e2e --no-cpu-baseline --no-e3 > /dev/null 2>&1
python scripts/launch_summary.py gpurun_out/r02_15_launches.csv | head -20
timeout 300 python bench.py --workload sgemm --steps 6 --no-e2e --no-cpu-baseline --no-e3 > /tmp/s.json 2> /tmp/s.err
tail -1 /tmp/s.json | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(round(d['value'],1), d['ms_per_step'], d['kernel_ms_avg'], d['kernel_timing'])"
