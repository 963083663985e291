python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || true
timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -q -x -k "push or tbk or heat or jacobi" 2>&1 | tail -2
r() { (cd $1 && timeout 600 python bench.py $2 --steps 10 --warmup 3 --no-e2e --no-cpu-baseline > /tmp/b.log 2>&1; tail -1 /tmp/b.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$1 $2', round(d['value'],1), round(d['roofline']['frac'],3), d['clocks']['sm_mhz'], d['clocks']['power_w_max'])"); }
r ab_old ""; r . ""; r ab_old "--workload heat3d"; r . "--workload heat3d"; r . "--parts 8 --push"; r . "--variant hotspot2d"
