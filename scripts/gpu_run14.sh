timeout 300 python scripts/graph_debug.py 2>&1 | tail -4
timeout 900 python -m pytest tests -m gpu -q -x 2>&1 | tail -5
timeout 300 python bench.py --workload jacobi2d --parts 8 --no-cpu-baseline --no-e2e > gpurun_out/bench_jacobi_p8.log 2>&1; tail -c 800 gpurun_out/bench_jacobi_p8.log; echo
timeout 300 python bench.py --parts 8 --steps 3 --no-cpu-baseline --no-e2e --abg > gpurun_out/bench_hot_p8.log 2>&1; tail -c 1200 gpurun_out/bench_hot_p8.log; echo
timeout 300 python bench.py --workload heat3d --parts 8 --steps 3 --no-cpu-baseline --no-e2e > gpurun_out/bench_heat_p8.log 2>&1; tail -c 800 gpurun_out/bench_heat_p8.log; echo
