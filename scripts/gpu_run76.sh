# hotspot2d_tbk: consumer warps per CTA x CTAs per SM (NW, MINB) on one box
run() {
  PK_NVCC_FLAGS="-DPK_TBK_NW=$1 -DPK_TBK_MINB=$2" python -c "from paper_conf_icppw_matzdf20_b200 import build; build.build(force=True)" > gpurun_out/build.log 2>&1 || tail -5 gpurun_out/build.log
  export PK_TBK_NW=$1
  timeout 300 python bench.py --steps 10 --warmup 3 --no-e2e --no-cpu-baseline > /tmp/b.log 2>&1; tail -1 /tmp/b.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('NW=$1 MINB=$2', round(d['value'],1), round(d['roofline']['frac'],3), round(d['kernel_ms_avg'],4), d['clocks']['sm_mhz'])" || tail -3 /tmp/b.log
}
run 4 3; run 3 4; run 4 3; run 3 4
PK_TBK_NW=3 timeout 600 python -m pytest tests/test_gpu_parity.py -m gpu -q -x -k "tbk" 2>&1 | tail -1
