timeout 900 python -m pytest tests -m gpu -q -x 2>&1 | tail -15
timeout 300 python bench.py --workload jacobi2d --parts 8 --no-cpu-baseline --no-e2e > gpurun_out/bench_jacobi_p8.log 2>&1; tail -c 700 gpurun_out/bench_jacobi_p8.log; echo
timeout 300 python bench.py --parts 8 --steps 3 --no-cpu-baseline --no-e2e > gpurun_out/bench_hot_p8.log 2>&1; tail -c 700 gpurun_out/bench_hot_p8.log; echo
