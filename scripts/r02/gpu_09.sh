# round 2, call 9: GEMM v2 converter (LDS/STS, native F2FP.TF32): GEMM tests + bench P=1; then the stencil A/B
timeout 900 python -m pytest tests -m gpu -q -x -k "gemm or sgemm or c4" > gpurun_out/r02_09_gemm.log 2>&1; echo "gemm tests: $(tail -1 gpurun_out/r02_09_gemm.log)"
grep -E "^E |FAILED" gpurun_out/r02_09_gemm.log | head -20
timeout 300 python bench.py --workload sgemm --steps 6 --no-e2e --no-cpu-baseline --no-e3 > /tmp/s.json 2> /tmp/s.err
tail -1 /tmp/s.json | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('sgemm P1', round(d['value'],1), round(d['ms_per_step'],2), 'frac', round(d['roofline']['frac'],3), d['clocks']['sm_mhz'], d['clocks']['reasons'])" || tail -5 /tmp/s.err
bash scripts/r02/gpu_08.sh
