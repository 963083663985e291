# round 2, call 57: heat3d_tb3 with column-edge templates: parity, then burst (10 steps) and sustained
# (60 steps, ~2.5 s) C3 throughput of tb2 vs tb3 in alternation, board power from the bench's sampler
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r02_57_build.log 2>&1 || tail -5 gpurun_out/r02_57_build.log
timeout 300 python -m pytest tests/test_gpu_parity.py -q -x -k "heat3d_tb3" > gpurun_out/r02_57_pytest.log 2>&1; rc=$?; echo "tb3 parity rc=$rc: $(tail -1 gpurun_out/r02_57_pytest.log)"
[ $rc -ne 0 ] && exit 0
run() {
  timeout 300 python bench.py --workload heat3d --iters 48 --no-e2e --no-cpu-baseline --no-e3 $2 > /tmp/b.json 2> /tmp/b.err
  tail -1 /tmp/b.json | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$1', round(d['value'],1), 'frac', round(d['roofline']['frac'],4), 'kms', round(d['kernel_ms_avg'],4), 'ms/step', round(d['ms_per_step'],2), d['clocks']['sm_mhz'], d['clocks']['reasons'], d['clocks'].get('power_w_max'))" || tail -3 /tmp/b.err
}
T="--variant heat3d_tb3 --tile 64"
for r in 1 2; do
  run "tb2 burst     " "--steps 10"
  run "tb3 burst     " "$T --steps 10"
  run "tb2 sustained " "--steps 60"
  run "tb3 sustained " "$T --steps 60"
done
