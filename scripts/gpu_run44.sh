python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || true
for i in 1 2; do
timeout 600 python bench.py --workload heat3d --steps 5 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/b.log 2>&1; tail -1 gpurun_out/b.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(d['metric'], round(d['value'],1), round(d['roofline']['frac'],3), d['clocks']['sm_mhz'], d['clocks']['power_w_max'])"
timeout 600 python bench.py --steps 10 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/b.log 2>&1; tail -1 gpurun_out/b.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(d['metric'], round(d['value'],1), round(d['roofline']['frac'],3), d['clocks']['sm_mhz'], d['clocks']['power_w_max'])"
done
nvidia-smi --query-gpu=name,clocks.max.mem,clocks.mem,power.limit,temperature.gpu --format=csv
