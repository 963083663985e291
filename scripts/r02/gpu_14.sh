# round 2, call 14: GEMM variants at full size: v1 (split pre-pass) vs v3 (CTA pairs, on-chip split) 6 / 7 stages
KD=paper_conf_icppw_matzdf20_b200/csrc/kernels
for r in 1 2; do
for v in v1 v3_s6 v3_s7; do
  cp scratch/sgemm_$v.cu $KD/sgemm_tc.cu
  python -m paper_conf_icppw_matzdf20_b200.build > /tmp/bld.log 2>&1 || { echo BUILD FAIL $v; tail -5 /tmp/bld.log; continue; }
  timeout 300 python bench.py --workload sgemm --steps 6 --no-e2e --no-cpu-baseline --no-e3 > /tmp/s.json 2> /tmp/s.err
  tail -1 /tmp/s.json | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$v', round(d['value'],1), round(d['ms_per_step'],2), round(d['kernel_ms_avg'],2), d['clocks']['sm_mhz'], d['clocks']['reasons'])" || tail -3 /tmp/s.err
done
done
