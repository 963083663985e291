# round 2, call 73: final checkpoint (jacobi2d_tb C1 default, push runs 16, heat3d_tb3 variant) -- full GPU suite, build + smoke,
# every bench line, reference arm, N = 2 torchrun line, C2 launch list
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r02_73_build.log 2>&1 || tail -5 gpurun_out/r02_73_build.log
timeout 2400 python -m pytest tests -m gpu -q -x > gpurun_out/r02_73_pytest_gpu.log 2>&1; echo "gpu suite: $(tail -1 gpurun_out/r02_73_pytest_gpu.log)"
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r02_73_smoke.log 2>&1; tail -1 gpurun_out/r02_73_smoke.log
for w in hotspot2d heat3d sgemm nbody jacobi2d; do
  timeout 900 python bench.py --workload $w > gpurun_out/r02_73_$w.json 2> gpurun_out/r02_73_$w.err
  tail -1 gpurun_out/r02_73_$w.json | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$w', round(d['value'],1), d['unit'], 'frac', round((d.get('roofline') or {}).get('frac',0),4), 'e2e', round((d.get('e2e') or {}).get('value',0),1), 'host', round(d['host_us_per_launch'],2), 'E3', (d.get('e3_single_gpu_slowdown') or {}).get('slowdown_pct'), d['clocks']['sm_mhz'], d['clocks']['reasons'])" || tail -3 gpurun_out/r02_73_$w.err
done
timeout 600 python bench.py --impl reference --steps 3 --warmup 3 > gpurun_out/r02_73_reference.json 2>&1; tail -c 300 gpurun_out/r02_73_reference.json; echo
timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29573 bench.py --gpus 2 --steps 5 --warmup 3 > gpurun_out/r02_73_n2.json 2> gpurun_out/r02_73_n2.err; tail -c 400 gpurun_out/r02_73_n2.json; echo
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/r02_73_launches_c2.csv python bench.py --steps 2 --warmup 3 --no-e2e --no-cpu-baseline --no-e3 > /dev/null 2>&1
python scripts/launch_summary.py gpurun_out/r02_73_launches_c2.csv "python bench.py --steps 2 --warmup 3 --no-e2e --no-cpu-baseline --no-e3" | head -8
