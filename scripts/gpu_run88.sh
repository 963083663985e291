# N-body: sources per shared-memory tile (barriers per chunk) at 2 CTAs/SM, unroll 32
for t in 256 512 1024 256; do
PK_NVCC_FLAGS="-DPK_NBODY_TILE=$t" python -c "from paper_conf_icppw_matzdf20_b200 import build; build.build(force=True)" > gpurun_out/build.log 2>&1 || tail -5 gpurun_out/build.log
timeout 600 python bench.py --workload nbody --steps 2 --warmup 2 --no-e2e --no-cpu-baseline > /tmp/b.log 2>&1; tail -1 /tmp/b.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('tile=$t', round(d['value'],1), round(d['roofline']['frac'],3), round(d['kernel_ms_avg'],2), d['clocks']['sm_mhz'])" || tail -3 /tmp/b.log
done
