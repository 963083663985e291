timeout 1200 python -m pytest tests -m gpu -q 2>&1 | tail -30 > gpurun_out/pytest_gpu.log
for wl in heat3d nbody jacobi2d; do timeout 600 python bench.py --workload $wl --no-cpu-baseline > gpurun_out/bench_$wl.log 2>&1; done
timeout 600 python bench.py --parts 8 --no-cpu-baseline --no-e2e > gpurun_out/bench_hotspot_p8.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:heat -s 5 -c 1 -o gpurun_out/prof_heat python bench.py --workload heat3d --steps 1 --warmup 1 --iters 4 --no-e2e --no-cpu-baseline > gpurun_out/prof_heat.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:nbody -s 2 -c 1 -o gpurun_out/prof_nbody python bench.py --workload nbody --steps 1 --warmup 1 --iters 1 --no-e2e --no-cpu-baseline > gpurun_out/prof_nbody.log 2>&1
cat gpurun_out/pytest_gpu.log; tail -1 gpurun_out/bench_*.log
