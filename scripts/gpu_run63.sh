# A/B on one box: mbarrier try_wait with a suspend-time hint (default) vs plain spin (PK_*_SPIN)
for fl in "" "-DPK_HEATTB_SPIN -DPK_TBK_SPIN" "" "-DPK_HEATTB_SPIN -DPK_TBK_SPIN"; do
PK_NVCC_FLAGS="$fl" python -c "from paper_conf_icppw_matzdf20_b200 import build; build.build(force=True)" > gpurun_out/build.log 2>&1 || tail -5 gpurun_out/build.log
for a in "--workload heat3d" ""; do
timeout 300 python bench.py $a --steps 5 --warmup 3 --no-e2e --no-cpu-baseline > /tmp/b.log 2>&1; tail -1 /tmp/b.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('[$fl] $a', round(d['value'],1), round(d['roofline']['frac'],3), round(d['kernel_ms_avg'],4), d['clocks']['sm_mhz'], d['clocks']['reasons'])" || tail -3 /tmp/b.log
done
done
python -c "from paper_conf_icppw_matzdf20_b200 import build; build.build(force=True)" > gpurun_out/build.log 2>&1
timeout 600 python -m pytest tests/test_gpu_parity.py -m gpu -q -x -k "heat3d_tb2 or tbk" 2>&1 | tail -1
timeout 400 ncu --set full --clock-control none --import-source on -k regex:heat -s 5 -c 1 -o gpurun_out/prof_heat_tb2_sleep python bench.py --workload heat3d --steps 1 --warmup 1 --iters 12 --no-e2e --no-cpu-baseline > gpurun_out/prof_heat_tb2_sleep.log 2>&1
