timeout 300 python -m pytest tests/test_gpu_parity.py -m gpu -q -x -k "heat or nbody" 2>&1 | tail -15 > gpurun_out/pytest_hn.log
cat gpurun_out/pytest_hn.log
timeout 300 python bench.py --workload heat3d --no-cpu-baseline --no-e2e > gpurun_out/bench_heat3d.log 2>&1
tail -c 500 gpurun_out/bench_heat3d.log; echo
timeout 300 python bench.py --workload nbody --steps 3 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/bench_nbody.log 2>&1
tail -c 500 gpurun_out/bench_nbody.log; echo
for ty in 32 128; do timeout 300 python bench.py --tile $ty --no-cpu-baseline --no-e2e > gpurun_out/bench_hot_ty$ty.log 2>&1; tail -c 400 gpurun_out/bench_hot_ty$ty.log; echo; done
timeout 400 ncu --set full --clock-control none --import-source on -k regex:heat -s 5 -c 1 -o gpurun_out/prof_heat7 python bench.py --workload heat3d --steps 1 --warmup 1 --iters 4 --no-e2e --no-cpu-baseline > gpurun_out/prof_heat7.log 2>&1
