# round 2, call 53: heat3d_tb3 skewed loop (S1 of the next plane after S2/S3 in one barrier interval) vs
# the plain order; parity first
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r02_53_build.log 2>&1 || tail -5 gpurun_out/r02_53_build.log
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "heat3d_tb3" > gpurun_out/r02_53_pytest.log 2>&1; echo "tb3 parity: $(tail -1 gpurun_out/r02_53_pytest.log)"
run() {
  PK_NVCC_FLAGS="$3" python -m paper_conf_icppw_matzdf20_b200.build > /dev/null 2>&1 || echo BUILD FAIL $3
  timeout 300 python bench.py --workload heat3d --iters 48 --steps 10 --no-e2e --no-cpu-baseline --no-e3 $2 > /tmp/b.json 2> /tmp/b.err
  tail -1 /tmp/b.json | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$1', round(d['value'],1), 'frac', round(d['roofline']['frac'],4), 'kms', round(d['kernel_ms_avg'],4), d['clocks']['sm_mhz'], d['clocks']['reasons'], d['clocks'].get('power_w_max'))" || tail -3 /tmp/b.err
}
for r in 1 2; do
  run "tb2 zc64      " "" ""
  run "tb3 skew zc64 " "--variant heat3d_tb3 --tile 64" ""
  run "tb3 plain zc64" "--variant heat3d_tb3 --tile 64" "-DPK_HEATTB3_SKEW=0"
  run "tb3 skew ns4  " "--variant heat3d_tb3 --tile 64" "-DPK_HEATTB3_NS=4"
done
python -m paper_conf_icppw_matzdf20_b200.build > /dev/null 2>&1
mkdir -p gpurun_out/r02_53
python bench.py --workload heat3d --iters 48 --steps 2 --warmup 3 --no-e2e --no-cpu-baseline --no-e3 --variant heat3d_tb3 --tile 64 > gpurun_out/r02_53_plain.log 2>&1 &&
timeout 600 ncu --set full --clock-control none --import-source on -k regex:heat3d_tb3 -s 5 -c 1 -o gpurun_out/r02_53/tb3 python bench.py --workload heat3d --iters 48 --steps 2 --warmup 3 --no-e2e --no-cpu-baseline --no-e3 --variant heat3d_tb3 --tile 64 > /dev/null 2>&1; echo ncu rc $?
