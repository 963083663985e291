python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || true
python scripts/gemm_err_scaling.py 2>&1 | tail -4
timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -q -x -k "gemm or sgemm" 2>&1 | tail -2
timeout 900 python -m pytest tests/test_gpu_fullsize.py -m gpu -q -x -k "sgemm or nbody" 2>&1 | tail -4
timeout 300 python bench.py --workload sgemm --no-e2e --no-cpu-baseline --steps 3 --warmup 3 > gpurun_out/b.log 2>&1; tail -1 gpurun_out/b.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(d['value'], d['roofline']['frac'], d['kernel_ms_avg'])"
