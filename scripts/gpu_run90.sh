# heat3d_tb2: float2 lanes (60-column blocks, fewer registers, more CTAs/SM) vs float4
run() {  # V MINB NS
  PK_NVCC_FLAGS="-DPK_HEATTB_V=$1 -DPK_HEATTB_MINB=$2 -DPK_HEATTB_NS=$3" python -c "from paper_conf_icppw_matzdf20_b200 import build; build.build(force=True)" > gpurun_out/build.log 2>&1 || tail -5 gpurun_out/build.log
  export PK_HEATTB_COLS=$((30 * $1))
  timeout 300 python bench.py --workload heat3d --steps 5 --warmup 3 --no-e2e --no-cpu-baseline > /tmp/b.log 2>&1; tail -1 /tmp/b.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('V=$1 MINB=$2 NS=$3', round(d['value'],1), round(d['roofline']['frac'],3), round(d['kernel_ms_avg'],4), d['clocks']['sm_mhz'])" || tail -3 /tmp/b.log
}
run 2 4 6
PK_HEATTB_COLS=60 timeout 600 python -m pytest tests/test_gpu_parity.py -m gpu -q -x -k "heat3d_tb2" 2>&1 | tail -1
run 4 3 6; run 2 4 8; run 2 5 6; run 2 5 8; run 2 3 6; run 4 3 6; run 2 4 6
