# round 2, call 22: full GPU suite after the C2 tile change
timeout 1500 python -m pytest tests -m gpu -q -x > gpurun_out/r02_22_pytest.log 2>&1; echo "gpu suite: $(tail -1 gpurun_out/r02_22_pytest.log)"
grep -E "^E |FAILED" gpurun_out/r02_22_pytest.log | head -10
