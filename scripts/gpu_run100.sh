# heat3d_tb2 register cap: HEAD (__launch_bounds__(160, 3) -> 128 regs, spills in the loop) vs __maxnreg__(136)
# (3 CTAs still fit: 15 warps x 17 allocation units), with 64-bit (i64) or 32-bit (i32) row/plane indices
K=paper_conf_icppw_matzdf20_b200/csrc/kernels/heat_tb.cu
cp $K /tmp/heat_tb_keep.cu
run() {
  cp scripts/heat_variants/heat_tb_$1.cu $K
  PK_NVCC_FLAGS="$2" python -c "from paper_conf_icppw_matzdf20_b200 import build; build.build(force=True)" > gpurun_out/build.log 2>&1 || tail -5 gpurun_out/build.log
  timeout 300 python bench.py --workload heat3d --steps 5 --warmup 3 --no-e2e --no-cpu-baseline > /tmp/b.log 2>&1; tail -1 /tmp/b.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$1 $2', round(d['value'],1), round(d['roofline']['frac'],3), round(d['kernel_ms_avg'],4), d['clocks']['sm_mhz'], d['clocks']['reasons'])" || tail -3 /tmp/b.log
}
for r in 1 2; do
run head ""; run i64 "-DPK_HEATTB_MAXNREG=136"; run i32 "-DPK_HEATTB_MAXNREG=136"; run i32 "-DPK_HEATTB_MAXNREG=128"
done
cp /tmp/heat_tb_keep.cu $K
