# round 2, call 10: ncu --set full of GEMM v2 (4096 x 4096 x 16384, one launch), streamed test
timeout 600 ncu --set full --clock-control none --import-source on -k regex:k_sgemm -c 1 -o gpurun_out/r02_sgemm_v2 python scripts/gemm_debug.py 4096x4096x16384 > gpurun_out/r02_10_ncu.log 2>&1; tail -3 gpurun_out/r02_10_ncu.log
python scripts/ncu_summary.py gpurun_out/r02_sgemm_v2.ncu-rep > gpurun_out/r02_sgemm_v2_summary.txt 2>&1; cat gpurun_out/r02_sgemm_v2_summary.txt | head -40
timeout 600 python -m pytest tests/test_gpu_parity.py -q -x -k "streamed" 2>&1 | tail -3
