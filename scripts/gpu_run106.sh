# heat3d_tb2 (32-bit indices): ring depth NS and producer back-off PNS re-checked
run() {
  PK_NVCC_FLAGS="$1" python -c "from paper_conf_icppw_matzdf20_b200 import build; build.build(force=True)" > gpurun_out/build.log 2>&1 || tail -5 gpurun_out/build.log
  timeout 300 python bench.py --workload heat3d --steps 5 --warmup 3 --no-e2e --no-cpu-baseline > /tmp/b.log 2>&1; tail -1 /tmp/b.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('[$1]', round(d['value'],1), round(d['roofline']['frac'],3), round(d['kernel_ms_avg'],4), d['clocks']['sm_mhz'], d['clocks']['reasons'])" || tail -3 /tmp/b.log
}
for r in 1 2; do
run ""; run "-DPK_HEATTB_NS=7"; run "-DPK_HEATTB_NS=5"; run "-DPK_HEATTB_PNS=128"; run "-DPK_HEATTB_PNS=512"
done
