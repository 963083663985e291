timeout 300 python -m pytest tests/test_gpu_parity.py -m gpu -q -x -k "tb2" 2>&1 | tail -15
timeout 300 python bench.py --variant hotspot2d_tb2 --no-cpu-baseline --no-e2e > gpurun_out/bench_hot_tb2.log 2>&1; tail -c 900 gpurun_out/bench_hot_tb2.log; echo
timeout 400 ncu --set full --clock-control none --import-source on -k regex:tb2 -s 5 -c 1 -o gpurun_out/prof_hotspot_tb2 python bench.py --variant hotspot2d_tb2 --steps 1 --warmup 1 --iters 10 --no-e2e --no-cpu-baseline > /dev/null 2>&1
