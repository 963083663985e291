# round 2, call 78: random launch programs on tile partitions (strided halo copies)
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r02_78_build.log 2>&1 || tail -5 gpurun_out/r02_78_build.log
timeout 900 python -m pytest tests/test_gpu_parity.py -q -k "random_launch" > gpurun_out/r02_78_pytest.log 2>&1; echo "random programs: $(tail -1 gpurun_out/r02_78_pytest.log)"
grep -E "^E |FAILED" gpurun_out/r02_78_pytest.log | head -8
