timeout 300 python -m pytest tests/test_gpu_parity.py -m gpu -q -x -k "tb2 or nbody" 2>&1 | tail -3
timeout 300 python bench.py --variant hotspot2d_tb2 --no-cpu-baseline --no-e2e > gpurun_out/bench_hot_tb2.log 2>&1; python -c "
import json; d=json.loads(open('gpurun_out/bench_hot_tb2.log').read().strip().splitlines()[-1]); print('tb2', d['value'], d['ms_per_step'], d['roofline']['frac'], d['kernel_ms_avg'])"
timeout 400 ncu --set full --clock-control none --import-source on -k regex:tb2 -s 5 -c 1 -o gpurun_out/prof_hotspot_tb2c python bench.py --variant hotspot2d_tb2 --steps 1 --warmup 1 --iters 10 --no-e2e --no-cpu-baseline > /dev/null 2>&1
