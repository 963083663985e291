python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || true
timeout 1500 python -m pytest tests -m gpu -q > gpurun_out/pytest_gpu.log 2>&1; echo "PYTEST: $(tail -1 gpurun_out/pytest_gpu.log)"
grep -E "FAILED|Error" gpurun_out/pytest_gpu.log | head -5
