# round 2, call 16: GEMM v3 with relaxed remote arrivals vs v1
KD=paper_conf_icppw_matzdf20_b200/csrc/kernels
for v in v3_relaxed v1 v3_relaxed; do
  cp scratch/sgemm_$v.cu $KD/sgemm_tc.cu
  python -m paper_conf_icppw_matzdf20_b200.build > /tmp/bld.log 2>&1 || { echo BUILD FAIL $v; tail -5 /tmp/bld.log; continue; }
  timeout 300 python bench.py --workload sgemm --steps 6 --no-e2e --no-cpu-baseline --no-e3 > /tmp/s.json 2> /tmp/s.err
  tail -1 /tmp/s.json | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$v', round(d['value'],1), round(d['ms_per_step'],2), d['clocks']['sm_mhz'], d['clocks']['reasons'])" || tail -3 /tmp/s.err
done
timeout 300 python scripts/gemm_debug.py 256x256x512 640x520x2048 2048x2048x16384
