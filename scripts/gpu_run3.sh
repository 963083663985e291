timeout 1200 python -m pytest tests -m gpu -q -x 2>&1 | tail -30 > gpurun_out/pytest_gpu.log
timeout 600 python bench.py --no-cpu-baseline --no-e2e > gpurun_out/bench_hotspot_tma.log 2>&1
timeout 600 python bench.py --no-cpu-baseline --no-e2e --variant hotspot2d_regs > gpurun_out/bench_hotspot_regs.log 2>&1
timeout 600 python bench.py --workload heat3d --no-cpu-baseline --no-e2e > gpurun_out/bench_heat3d.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:hotspot -s 10 -c 1 -o gpurun_out/prof_hotspot_tma python bench.py --steps 1 --warmup 1 --iters 10 --no-e2e --no-cpu-baseline > gpurun_out/prof_hotspot_tma.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:heat -s 5 -c 1 -o gpurun_out/prof_heat2 python bench.py --workload heat3d --steps 1 --warmup 1 --iters 4 --no-e2e --no-cpu-baseline > gpurun_out/prof_heat2.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:nbody -s 1 -c 1 -o gpurun_out/prof_nbody python bench.py --workload nbody --steps 1 --warmup 1 --iters 1 --no-e2e --no-cpu-baseline > gpurun_out/prof_nbody.log 2>&1
cat gpurun_out/pytest_gpu.log
for f in gpurun_out/bench_hotspot_tma.log gpurun_out/bench_hotspot_regs.log gpurun_out/bench_heat3d.log; do tail -n 1 $f | cut -c1-600; done
