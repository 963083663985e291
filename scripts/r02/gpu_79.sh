# round 2, call 79: SPMD peer-memory processes (2 and 3 ranks on one GPU, stream-memop and SM flags) with the
# random launch programs added to the worker
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r02_79_build.log 2>&1 || tail -5 gpurun_out/r02_79_build.log
timeout 1200 python -m pytest tests/test_gpu_spmd_ipc.py -q > gpurun_out/r02_79_pytest.log 2>&1; echo "spmd ipc: $(tail -1 gpurun_out/r02_79_pytest.log)"
grep -E "^E |FAILED|AssertionError" gpurun_out/r02_79_pytest.log | head -8
