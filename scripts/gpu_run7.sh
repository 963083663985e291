timeout 300 python -m pytest tests/test_gpu_parity.py -m gpu -q -x -k "heat or gemm" 2>&1 | tail -15 > gpurun_out/pytest_hg.log
cat gpurun_out/pytest_hg.log
timeout 300 python bench.py --workload heat3d --no-cpu-baseline --no-e2e > gpurun_out/bench_heat3d.log 2>&1
tail -c 600 gpurun_out/bench_heat3d.log; echo
timeout 600 python bench.py --workload sgemm --steps 5 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/bench_sgemm.log 2>&1
tail -c 800 gpurun_out/bench_sgemm.log; echo
timeout 600 ncu --set full --clock-control none --import-source on -k regex:sgemm -s 3 -c 1 -o gpurun_out/prof_sgemm2 python bench.py --workload sgemm --steps 1 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/prof_sgemm2.log 2>&1
timeout 400 ncu --set full --clock-control none --import-source on -k regex:heat -s 5 -c 1 -o gpurun_out/prof_heat6 python bench.py --workload heat3d --steps 1 --warmup 1 --iters 4 --no-e2e --no-cpu-baseline > gpurun_out/prof_heat6.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:nbody_partial -s 3 -c 1 -o gpurun_out/prof_nbody3 python bench.py --workload nbody --steps 1 --warmup 3 --iters 1 --no-e2e --no-cpu-baseline > gpurun_out/prof_nbody3.log 2>&1
