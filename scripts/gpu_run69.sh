# N-body source split: work items per step (tail of the persistent grid)
for sp in 8 16 32 8; do
PK_NVCC_FLAGS="-DPK_NBODY_SPLIT=$sp" python -c "from paper_conf_icppw_matzdf20_b200 import build; build.build(force=True)" > gpurun_out/build.log 2>&1 || tail -5 gpurun_out/build.log
timeout 600 python bench.py --workload nbody --steps 2 --warmup 3 --no-e2e --no-cpu-baseline > /tmp/b.log 2>&1; tail -1 /tmp/b.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('split=$sp', round(d['value'],1), round(d['roofline']['frac'],3), round(d['kernel_ms_avg'],2), d['clocks']['sm_mhz'], d['clocks']['reasons'])" || tail -3 /tmp/b.log
done
PK_NVCC_FLAGS="-DPK_NBODY_SPLIT=16" python -c "from paper_conf_icppw_matzdf20_b200 import build; build.build(force=True)" > gpurun_out/build.log 2>&1
timeout 600 python -m pytest tests/test_gpu_parity.py -m gpu -q -x -k "nbody" 2>&1 | tail -1
