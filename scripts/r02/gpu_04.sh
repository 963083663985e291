# round 2, call 4: copy-engine / capture probe; GEMM v2 (on-chip split, MN-major B, diagonal chunks) parity + bench
timeout 60 ./scripts/ce_probe.bin
timeout 900 python -m pytest tests -m gpu -q -x -k "gemm or sgemm or c4" > gpurun_out/r02_04_pytest.log 2>&1; echo "gemm tests: $(tail -1 gpurun_out/r02_04_pytest.log)"
grep -E "FAILED|Error|assert" gpurun_out/r02_04_pytest.log | head -20
timeout 300 python bench.py --workload sgemm --steps 5 --no-e2e --no-cpu-baseline --no-e3 > gpurun_out/r02_04_bench_sgemm.json 2> gpurun_out/r02_04_bench_sgemm.err
tail -1 gpurun_out/r02_04_bench_sgemm.json | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('sgemm', round(d['value'],1), d['roofline'], d['clocks'])" || tail -5 gpurun_out/r02_04_bench_sgemm.err
