# N-body: CTAs per SM (registers) x source unroll on one box
run() {
  PK_NVCC_FLAGS="-DPK_NBODY_MINB=$1 -DPK_NBODY_UNROLL=$2" python -c "from paper_conf_icppw_matzdf20_b200 import build; build.build(force=True)" > gpurun_out/build.log 2>&1 || tail -5 gpurun_out/build.log
  timeout 600 python bench.py --workload nbody --steps 2 --warmup 2 --no-e2e --no-cpu-baseline > /tmp/b.log 2>&1; tail -1 /tmp/b.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('MINB=$1 U=$2', round(d['value'],1), round(d['roofline']['frac'],3), round(d['kernel_ms_avg'],2), d['clocks']['sm_mhz'])" || tail -3 /tmp/b.log
}
run 2 32; run 2 64; run 2 128; run 2 32
