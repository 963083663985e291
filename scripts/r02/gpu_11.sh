# round 2, call 11: GEMM v2 with 10 converter warps (epilogue warps convert too)
timeout 900 python -m pytest tests -m gpu -q -x -k "gemm or sgemm or c4" > gpurun_out/r02_11_gemm.log 2>&1; echo "gemm tests: $(tail -1 gpurun_out/r02_11_gemm.log)"
grep -E "^E |FAILED" gpurun_out/r02_11_gemm.log | head -20
for P in 1 4; do
timeout 300 python bench.py --workload sgemm --parts $P --steps 6 --no-e2e --no-cpu-baseline --no-e3 > /tmp/s.json 2> /tmp/s.err
tail -1 /tmp/s.json | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('sgemm P$P', round(d['value'],1), round(d['ms_per_step'],2), 'frac', round(d['roofline']['frac'],3), d['transfers']['moved_bytes'], d['clocks']['sm_mhz'], d['clocks']['reasons'])" || tail -5 /tmp/s.err
done
timeout 600 ncu --set full --clock-control none --import-source on -k regex:k_sgemm -c 1 -o gpurun_out/r02_sgemm_v2b python scripts/gemm_debug.py 4096x4096x16384 > gpurun_out/r02_11_ncu.log 2>&1; tail -1 gpurun_out/r02_11_ncu.log
python scripts/ncu_summary.py gpurun_out/r02_sgemm_v2b.ncu-rep | grep -E "time|tensor|dram__bytes|issue"
