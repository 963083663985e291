# round 2, call 7: GEMM v2 + streamed B: GEMM tests, full GPU suite, bench P=1 / P=4 virtual (overlap on/off)
timeout 900 python -m pytest tests -m gpu -q -x -k "gemm or sgemm or c4" > gpurun_out/r02_07_gemm.log 2>&1; echo "gemm tests: $(tail -1 gpurun_out/r02_07_gemm.log)"
grep -E "FAILED|Error|assert" gpurun_out/r02_07_gemm.log | head -20
for P in 1 4; do
 for m in "" "--no-overlap"; do
  timeout 300 python bench.py --workload sgemm --parts $P --steps 6 --no-e2e --no-cpu-baseline --no-e3 $m > gpurun_out/r02_07_sgemm_$P$m.json 2> gpurun_out/r02_07_sgemm_$P$m.err
  tail -1 gpurun_out/r02_07_sgemm_$P$m.json | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('sgemm P$P $m', round(d['value'],1), round(d['ms_per_step'],2), 'frac', round(d['roofline']['frac'],3), d['transfers'], d['clocks']['sm_mhz'], d['clocks']['reasons'])" || tail -5 gpurun_out/r02_07_sgemm_$P$m.err
 done
done
timeout 1500 python -m pytest tests -m gpu -q -x > gpurun_out/r02_07_pytest.log 2>&1; echo "gpu suite: $(tail -1 gpurun_out/r02_07_pytest.log)"
grep -E "FAILED|Error" gpurun_out/r02_07_pytest.log | head -10
