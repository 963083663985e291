# round 2, call 17: full GPU suite with GEMM v3 (CTA pairs); ncu --set full of the full-size GEMM
timeout 1500 python -m pytest tests -m gpu -q -x > gpurun_out/r02_17_pytest.log 2>&1; echo "gpu suite: $(tail -1 gpurun_out/r02_17_pytest.log)"
grep -E "^E |FAILED" gpurun_out/r02_17_pytest.log | head -10
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_sgemm -c 1 -o gpurun_out/r02_sgemm_v3_full python scripts/gemm_debug.py 16384x16384x16384 > gpurun_out/r02_17_ncu.log 2>&1; tail -1 gpurun_out/r02_17_ncu.log
python scripts/ncu_summary.py gpurun_out/r02_sgemm_v3_full.ncu-rep > gpurun_out/r02_sgemm_v3_full_summary.txt; cat gpurun_out/r02_sgemm_v3_full_summary.txt
