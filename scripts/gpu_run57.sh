# hotspot2d_tbk K = 4/6/8: 3-slot windows, reordered update (default) vs chained update (PK_TBK_CHAIN)
for fl in "" "-DPK_TBK_CHAIN"; do
PK_NVCC_FLAGS="$fl" python -c "from paper_conf_icppw_matzdf20_b200 import build; build.build(force=True)" > gpurun_out/build.log 2>&1 || tail -5 gpurun_out/build.log
echo "flags: $fl"
timeout 300 python scripts/tbk_probe.py 2>&1 | tail -3
for k in 4 6; do
timeout 300 python bench.py --sweeps $k --iters 96 --steps 5 --warmup 3 --no-e2e --no-cpu-baseline > /tmp/b.log 2>&1; tail -1 /tmp/b.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('K=$k', round(d['value'],1), round(d['roofline']['frac'],3), round(d['kernel_ms_avg'],4), d['clocks']['sm_mhz'])" || tail -3 /tmp/b.log
done
done
