timeout 300 python -m pytest tests/test_gpu_parity.py -m gpu -q -x -k "heat or nbody" 2>&1 | tail -15 > gpurun_out/pytest_hn.log
cat gpurun_out/pytest_hn.log
timeout 300 python bench.py --workload heat3d --no-cpu-baseline --no-e2e > gpurun_out/bench_heat3d.log 2>&1
tail -c 450 gpurun_out/bench_heat3d.log; echo
timeout 300 python bench.py --workload heat3d --tile 256 --no-cpu-baseline --no-e2e > gpurun_out/bench_heat3d_zc256.log 2>&1
tail -c 450 gpurun_out/bench_heat3d_zc256.log; echo
timeout 400 ncu --set full --clock-control none --import-source on -k regex:heat -s 5 -c 1 -o gpurun_out/prof_heat8 python bench.py --workload heat3d --steps 1 --warmup 1 --iters 4 --no-e2e --no-cpu-baseline > gpurun_out/prof_heat8.log 2>&1
timeout 600 python bench.py --parts 8 --abg --no-cpu-baseline --no-e2e --steps 5 > gpurun_out/bench_hot_p8_abg.log 2>&1
tail -c 1500 gpurun_out/bench_hot_p8_abg.log; echo
