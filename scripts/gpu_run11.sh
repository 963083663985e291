timeout 900 python -m pytest tests -m gpu -q 2>&1 | tail -5 > gpurun_out/pytest_all.log; cat gpurun_out/pytest_all.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -2
timeout 600 python bench.py > gpurun_out/bench_default.log 2>&1; tail -n 1 gpurun_out/bench_default.log
timeout 300 python bench.py --workload nbody --steps 3 --warmup 3 --no-cpu-baseline > gpurun_out/bench_nbody.log 2>&1; tail -c 400 gpurun_out/bench_nbody.log; echo
timeout 300 python bench.py --workload heat3d > gpurun_out/bench_heat3d.log 2>&1; tail -c 300 gpurun_out/bench_heat3d.log; echo
timeout 600 python bench.py --workload sgemm --steps 5 > gpurun_out/bench_sgemm.log 2>&1; tail -c 300 gpurun_out/bench_sgemm.log; echo
timeout 300 python bench.py --workload jacobi2d --parts 2 --no-cpu-baseline > gpurun_out/bench_jacobi_p2.log 2>&1; tail -c 300 gpurun_out/bench_jacobi_p2.log; echo
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/launches_r01.csv python bench.py --steps 2 --warmup 1 --no-e2e --no-cpu-baseline > /dev/null 2>&1
timeout 600 python bench.py --impl reference --steps 3 --warmup 1 > gpurun_out/bench_reference.log 2>&1; tail -n 1 gpurun_out/bench_reference.log
