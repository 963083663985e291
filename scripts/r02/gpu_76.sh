# round 2, call 76: randomised launch programs (two kernels on shared ping-pong buffers, re-uploads,
# mid-program reads) at P = 3/4/5 in every ordering mode, bit-identical to P = 1
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r02_76_build.log 2>&1 || tail -5 gpurun_out/r02_76_build.log
timeout 900 python -m pytest tests/test_gpu_parity.py -q -k "random_launch" > gpurun_out/r02_76_pytest.log 2>&1; echo "random programs: $(tail -1 gpurun_out/r02_76_pytest.log)"
grep -E "^E |FAILED" gpurun_out/r02_76_pytest.log | head -8
