# hotspot2d_tbk: power-of-two ring stage stride vs packed, on one box
for fl in "" "-DPK_TBK_POW2" "" "-DPK_TBK_POW2"; do
PK_NVCC_FLAGS="$fl" python -c "from paper_conf_icppw_matzdf20_b200 import build; build.build(force=True)" > gpurun_out/build.log 2>&1 || tail -5 gpurun_out/build.log
timeout 300 python bench.py --steps 10 --warmup 3 --no-e2e --no-cpu-baseline > /tmp/b.log 2>&1; tail -1 /tmp/b.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('[$fl]', round(d['value'],1), round(d['roofline']['frac'],3), round(d['kernel_ms_avg'],4), d['clocks']['sm_mhz'])" || tail -3 /tmp/b.log
done
