# round 2, call 1: GPU suite after the pins / per-device attributes / scratch / memo / capture-fallback changes
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,power.draw,power.limit --format=csv > gpurun_out/r02_01_smi.txt 2>&1
timeout 1500 python -m pytest tests -m gpu -q -x --durations=15 > gpurun_out/r02_01_pytest.log 2>&1; echo "gpu suite: $(tail -1 gpurun_out/r02_01_pytest.log)"
tail -30 gpurun_out/r02_01_pytest.log
