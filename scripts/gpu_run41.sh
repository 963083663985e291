python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || true
free -g | head -2; nproc
timeout 1700 python -m pytest tests/test_gpu_fullsize.py -m gpu -q -x --durations=0 2>&1 | tail -25
