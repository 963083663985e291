# round 2, call 54: heat3d_tb3 warp-specialised (3 sweep-1 warps feeding 4 row warps through a shared
# sweep-1 plane ring): parity first (under timeout), then the C3 bench at 48 sweeps per step vs tb2
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r02_54_build.log 2>&1 || tail -5 gpurun_out/r02_54_build.log
timeout 300 python -m pytest tests/test_gpu_parity.py -q -x -k "heat3d_tb3" > gpurun_out/r02_54_pytest.log 2>&1; rc=$?; echo "tb3 parity rc=$rc: $(tail -1 gpurun_out/r02_54_pytest.log)"
grep -E "^E |FAILED" gpurun_out/r02_54_pytest.log | head -8
[ $rc -ne 0 ] && exit 0
run() {
  timeout 300 python bench.py --workload heat3d --iters 48 --steps 10 --no-e2e --no-cpu-baseline --no-e3 $2 > /tmp/b.json 2> /tmp/b.err
  tail -1 /tmp/b.json | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$1', round(d['value'],1), 'frac', round(d['roofline']['frac'],4), 'kms', round(d['kernel_ms_avg'],4), d['clocks']['sm_mhz'], d['clocks']['reasons'], d['clocks'].get('power_w_max'))" || tail -3 /tmp/b.err
}
for r in 1 2; do
  run "tb2 zc64   " ""
  run "tb3ws zc64 " "--variant heat3d_tb3 --tile 64"
  run "tb3ws zc128" "--variant heat3d_tb3 --tile 128"
  run "tb3ws zc32 " "--variant heat3d_tb3 --tile 32"
done
