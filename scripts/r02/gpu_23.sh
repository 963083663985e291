# round 2, call 23: GEMM K-start quantisation (fine diagonal vs eighths vs none): speed and DRAM bytes
KD=paper_conf_icppw_matzdf20_b200/csrc/kernels
for v in diag_fine diag8 diag1; do
  if [ $v = diag1 ]; then cp scratch/sgemm_diag8.cu $KD/sgemm_tc.cu; export PK_NVCC_FLAGS="-DPK_SGEMM_DIAG=1"; else cp scratch/sgemm_$v.cu $KD/sgemm_tc.cu; unset PK_NVCC_FLAGS; fi
  python -m paper_conf_icppw_matzdf20_b200.build > /tmp/bld.log 2>&1 || { echo BUILD FAIL $v; tail -5 /tmp/bld.log; continue; }
  for r in 1 2; do
  timeout 300 python bench.py --workload sgemm --steps 6 --no-e2e --no-cpu-baseline --no-e3 > /tmp/s.json 2> /tmp/s.err
  tail -1 /tmp/s.json | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$v', round(d['value'],1), round(d['ms_per_step'],2), d['clocks']['sm_mhz'], d['clocks']['reasons'])" || tail -3 /tmp/s.err
  done
  timeout 600 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum --clock-control none -k regex:k_sgemm -c 1 python scripts/gemm_debug.py 16384x16384x16384 2>&1 | grep -E "dram__bytes|duration" | head -3
done
unset PK_NVCC_FLAGS
