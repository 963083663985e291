timeout 300 python -m pytest tests/test_gpu_parity.py -m gpu -q -x -k "nbody" 2>&1 | tail -5
timeout 300 python bench.py --workload nbody --steps 3 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/bench_nbody.log 2>&1
tail -c 500 gpurun_out/bench_nbody.log; echo
timeout 600 ncu --set full --clock-control none --import-source on -k regex:nbody_partial -s 3 -c 1 -o gpurun_out/prof_nbody4 python bench.py --workload nbody --steps 1 --warmup 3 --iters 1 --no-e2e --no-cpu-baseline > gpurun_out/prof_nbody4.log 2>&1
