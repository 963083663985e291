timeout 300 python -m pytest tests/test_gpu_parity.py -m gpu -q -x -k "heat" 2>&1 | tail -15 > gpurun_out/pytest_heat.log
cat gpurun_out/pytest_heat.log
timeout 900 python -m pytest tests -m gpu -q -x -k "not heat" 2>&1 | tail -15 > gpurun_out/pytest_gpu.log
cat gpurun_out/pytest_gpu.log
timeout 300 python bench.py --workload heat3d --no-cpu-baseline --no-e2e > gpurun_out/bench_heat3d.log 2>&1
tail -c 700 gpurun_out/bench_heat3d.log
timeout 300 python bench.py --workload nbody --steps 3 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/bench_nbody.log 2>&1
tail -c 700 gpurun_out/bench_nbody.log
timeout 600 python bench.py --workload sgemm --steps 5 --warmup 3 --no-cpu-baseline > gpurun_out/bench_sgemm.log 2>&1
tail -c 1200 gpurun_out/bench_sgemm.log
timeout 600 ncu --set full --clock-control none --import-source on -k regex:sgemm -s 3 -c 1 -o gpurun_out/prof_sgemm python bench.py --workload sgemm --steps 1 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/prof_sgemm.log 2>&1
timeout 400 ncu --set full --clock-control none --import-source on -k regex:heat -s 5 -c 1 -o gpurun_out/prof_heat5 python bench.py --workload heat3d --steps 1 --warmup 1 --iters 4 --no-e2e --no-cpu-baseline > gpurun_out/prof_heat5.log 2>&1
