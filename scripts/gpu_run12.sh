timeout 600 compute-sanitizer --tool memcheck --error-exitcode 9 python scripts/sanitize_smoke.py > gpurun_out/sanitize_memcheck.log 2>&1; echo "memcheck rc=$?"; tail -5 gpurun_out/sanitize_memcheck.log
timeout 900 compute-sanitizer --tool racecheck --error-exitcode 9 python scripts/sanitize_smoke.py > gpurun_out/sanitize_racecheck.log 2>&1; echo "racecheck rc=$?"; tail -5 gpurun_out/sanitize_racecheck.log
timeout 300 python -m pytest tests/test_gpu_parity.py -m gpu -q -k placement 2>&1 | tail -2
timeout 300 python bench.py --workload jacobi2d --parts 8 --no-cpu-baseline --no-e2e > gpurun_out/bench_jacobi_p8.log 2>&1; tail -c 900 gpurun_out/bench_jacobi_p8.log; echo
timeout 300 python bench.py --workload jacobi2d --parts 1 --no-cpu-baseline --no-e2e > gpurun_out/bench_jacobi_p1.log 2>&1; tail -c 700 gpurun_out/bench_jacobi_p1.log; echo
timeout 300 python bench.py --parts 8 --steps 3 --no-cpu-baseline --no-e2e > gpurun_out/bench_hot_p8.log 2>&1; tail -c 900 gpurun_out/bench_hot_p8.log; echo
