# heat3d_tb2: v1 structure + COLEDGE template + power-of-two ring (NS = 8 / 4); ZC sweep
for ns in 8 4; do
PK_NVCC_FLAGS="-DPK_HEATTB_NS=$ns" python -c "from paper_conf_icppw_matzdf20_b200 import build; build.build(force=True)" > gpurun_out/build.log 2>&1 || tail -5 gpurun_out/build.log
[ $ns = 8 ] && timeout 600 python -m pytest tests/test_gpu_parity.py -m gpu -q -x -k "heat3d_tb2 or heat_tile" 2>&1 | tail -1
for zc in 128 64 32; do
timeout 300 python bench.py --workload heat3d --tile $zc --steps 5 --warmup 3 --no-e2e --no-cpu-baseline > /tmp/b.log 2>&1; tail -1 /tmp/b.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('NS=$ns ZC=$zc', round(d['value'],1), round(d['roofline']['frac'],3), round(d['kernel_ms_avg'],4), d['clocks']['sm_mhz'], d['clocks']['reasons'])" || tail -3 /tmp/b.log
done
done
