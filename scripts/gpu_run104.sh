# heat3d_tb2: column-edge specialisation (interior-column blocks skip the x-clamp selects) vs without
K=paper_conf_icppw_matzdf20_b200/csrc/kernels/heat_tb.cu
cp $K /tmp/heat_tb_keep.cu
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || tail -5 gpurun_out/build.log
timeout 900 python -m pytest tests -m gpu -x -q -k "heat" > gpurun_out/pytest_heat.log 2>&1; echo "cedge heat tests: $(tail -1 gpurun_out/pytest_heat.log)"
run() {
  cp scripts/heat_variants/heat_tb_$1.cu $K
  python -c "from paper_conf_icppw_matzdf20_b200 import build; build.build(force=True)" > gpurun_out/build.log 2>&1 || tail -5 gpurun_out/build.log
  timeout 300 python bench.py --workload heat3d --steps 5 --warmup 3 --no-e2e --no-cpu-baseline > /tmp/b.log 2>&1; tail -1 /tmp/b.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$1', round(d['value'],1), round(d['roofline']['frac'],3), round(d['kernel_ms_avg'],4), d['clocks']['sm_mhz'], d['clocks']['reasons'])" || tail -3 /tmp/b.log
}
for r in 1 2 3; do run i32; run i32_cedge; done
cp /tmp/heat_tb_keep.cu $K
