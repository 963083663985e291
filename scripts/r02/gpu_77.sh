# round 2, call 77: full GPU suite with the widened random-program test (5 seeds x 40 ops)
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r02_77_build.log 2>&1 || tail -5 gpurun_out/r02_77_build.log
timeout 1800 python -m pytest tests -m gpu -q > gpurun_out/r02_77_pytest_gpu.log 2>&1; echo "gpu suite: $(tail -1 gpurun_out/r02_77_pytest_gpu.log)"
grep -E "^E |FAILED" gpurun_out/r02_77_pytest_gpu.log | head -8
