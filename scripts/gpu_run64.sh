# A/B on one box: heat3d_tb2 v1 (committed) vs v2 (32-bit index math, incremental ring slots) at 6 and 5 consumer warps
KF=paper_conf_icppw_matzdf20_b200/csrc/kernels/heat_tb.cu
run() {  # $1 = source, $2 = consumer warps
  cp scripts/heat_tb_$1.cu.txt $KF
  PK_NVCC_FLAGS="-DPK_HEATTB_NW=$2" python -c "from paper_conf_icppw_matzdf20_b200 import build; build.build(force=True)" > gpurun_out/build.log 2>&1 || tail -5 gpurun_out/build.log
  export PK_HEATTB_ROWS=$((4 * $2))
  timeout 300 python bench.py --workload heat3d --steps 5 --warmup 3 --no-e2e --no-cpu-baseline > /tmp/b.log 2>&1; tail -1 /tmp/b.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$1 NW=$2', round(d['value'],1), round(d['roofline']['frac'],3), round(d['kernel_ms_avg'],4), d['clocks']['sm_mhz'], d['clocks']['reasons'])" || tail -3 /tmp/b.log
}
run v2 5
timeout 600 python -m pytest tests/test_gpu_parity.py -m gpu -q -x -k "heat3d_tb2" 2>&1 | tail -1
run v1 6; run v2 6; run v2 5; run v1 6; run v2 6; run v2 5
