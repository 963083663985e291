timeout 300 python -m pytest tests/test_gpu_parity.py -m gpu -q -x -k "hotspot or graph or caller" 2>&1 | tail -4
for ty in 64 128 512; do timeout 300 python bench.py --tile $ty --no-cpu-baseline --no-e2e > gpurun_out/bench_hot_ty$ty.log 2>&1; python -c "
import json; d=json.loads(open('gpurun_out/bench_hot_ty$ty.log').read().strip().splitlines()[-1]); print($ty, d['value'], d['roofline']['frac'], d['kernel_ms_avg'])"; done
timeout 400 ncu --set full --clock-control none --import-source on -k regex:hotspot -s 10 -c 1 -o gpurun_out/prof_hotspot_chunks python bench.py --steps 1 --warmup 1 --iters 10 --no-e2e --no-cpu-baseline > /dev/null 2>&1
