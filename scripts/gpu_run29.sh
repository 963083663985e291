python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || true
timeout 1200 python -m pytest tests/test_gpu_spmd_ipc.py -m gpu -q -x --durations=5 2>&1 | tail -12
