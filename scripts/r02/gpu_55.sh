# round 2, call 55: heat3d_tb3 warp-specialised with y-neighbour reuse in sweep 2: parity, bench vs tb2, ncu
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r02_55_build.log 2>&1 || tail -5 gpurun_out/r02_55_build.log
timeout 300 python -m pytest tests/test_gpu_parity.py -q -x -k "heat3d_tb3" > gpurun_out/r02_55_pytest.log 2>&1; rc=$?; echo "tb3 parity rc=$rc: $(tail -1 gpurun_out/r02_55_pytest.log)"
[ $rc -ne 0 ] && exit 0
run() {
  timeout 300 python bench.py --workload heat3d --iters 48 --steps 10 --no-e2e --no-cpu-baseline --no-e3 $2 > /tmp/b.json 2> /tmp/b.err
  tail -1 /tmp/b.json | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$1', round(d['value'],1), 'frac', round(d['roofline']['frac'],4), 'kms', round(d['kernel_ms_avg'],4), d['clocks']['sm_mhz'], d['clocks']['reasons'], d['clocks'].get('power_w_max'))" || tail -3 /tmp/b.err
}
for r in 1 2; do
  run "tb2 zc64   " ""
  run "tb3ws zc64 " "--variant heat3d_tb3 --tile 64"
done
mkdir -p gpurun_out/r02_55
python bench.py --workload heat3d --iters 48 --steps 2 --warmup 3 --no-e2e --no-cpu-baseline --no-e3 --variant heat3d_tb3 --tile 64 > gpurun_out/r02_55_plain.log 2>&1 &&
timeout 600 ncu --set full --clock-control none --import-source on -k regex:heat3d_tb3 -s 5 -c 1 -o gpurun_out/r02_55/tb3ws python bench.py --workload heat3d --iters 48 --steps 2 --warmup 3 --no-e2e --no-cpu-baseline --no-e3 --variant heat3d_tb3 --tile 64 > /dev/null 2>&1; echo ncu rc $?
