# heat3d_tb2 with the producer back-off: consumer warps x CTAs/SM again (NW, MINB, NS)
run() {
  PK_NVCC_FLAGS="-DPK_HEATTB_NW=$1 -DPK_HEATTB_MINB=$2 -DPK_HEATTB_NS=$3" python -c "from paper_conf_icppw_matzdf20_b200 import build; build.build(force=True)" > gpurun_out/build.log 2>&1 || tail -5 gpurun_out/build.log
  export PK_HEATTB_ROWS=$((4 * $1))
  timeout 300 python bench.py --workload heat3d --steps 5 --warmup 3 --no-e2e --no-cpu-baseline > /tmp/b.log 2>&1; tail -1 /tmp/b.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('NW=$1 MINB=$2 NS=$3', round(d['value'],1), round(d['roofline']['frac'],3), round(d['kernel_ms_avg'],4), d['clocks']['sm_mhz'])" || tail -3 /tmp/b.log
}
run 4 3 6; run 3 4 6; run 2 6 6; run 4 3 6; run 3 4 6; run 2 6 6
