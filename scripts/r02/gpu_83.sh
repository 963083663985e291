# round 2, call 83: C1 kernels bit-exact against the fp32 CPU mirror (optional strong pin)
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r02_83_build.log 2>&1 || tail -5 gpurun_out/r02_83_build.log
timeout 900 python -m pytest tests/test_gpu_parity.py -q -k "fp32_cpu_mirror" > gpurun_out/r02_83_pytest.log 2>&1; echo "mirror: $(tail -1 gpurun_out/r02_83_pytest.log)"
grep -E "^E |FAILED" gpurun_out/r02_83_pytest.log | head -6
