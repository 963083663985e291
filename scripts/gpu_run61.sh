# A/B on one box: heat3d_tb2 committed (v1) vs COLEDGE + 8-slot ring
K=paper_conf_icppw_matzdf20_b200/csrc/kernels/heat_tb.cu
for v in v1 new v1 new; do
cp scripts/heat_tb_$v.cu.txt $K
python -c "from paper_conf_icppw_matzdf20_b200 import build; build.build()" > gpurun_out/build.log 2>&1 || tail -5 gpurun_out/build.log
for zc in 128 64; do
timeout 300 python bench.py --workload heat3d --tile $zc --steps 5 --warmup 3 --no-e2e --no-cpu-baseline > /tmp/b.log 2>&1; tail -1 /tmp/b.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$v ZC=$zc', round(d['value'],1), round(d['roofline']['frac'],3), round(d['kernel_ms_avg'],4), d['clocks']['sm_mhz'], d['clocks']['reasons'])" || tail -3 /tmp/b.log
done
done
