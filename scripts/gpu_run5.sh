timeout 900 python -m pytest tests -m gpu -q -x -k "not gemm" 2>&1 | tail -15 > gpurun_out/pytest_gpu.log
timeout 300 python -m pytest tests -m gpu -q -x -k "gemm" 2>&1 | tail -40 > gpurun_out/pytest_gemm.log
timeout 600 python bench.py --workload heat3d --no-cpu-baseline --no-e2e > gpurun_out/bench_heat3d.log 2>&1
timeout 600 python bench.py --workload heat3d --variant heat3d_regs --no-cpu-baseline --no-e2e > gpurun_out/bench_heat3d_regs.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:heat -s 5 -c 1 -o gpurun_out/prof_heat4 python bench.py --workload heat3d --steps 1 --warmup 1 --iters 4 --no-e2e --no-cpu-baseline > gpurun_out/prof_heat4.log 2>&1
cat gpurun_out/pytest_gpu.log gpurun_out/pytest_gemm.log
for f in gpurun_out/bench_heat3d.log gpurun_out/bench_heat3d_regs.log; do tail -n 1 $f | cut -c1-200; done
