timeout 300 python -m pytest tests/test_gpu_parity.py -m gpu -q -x -k "hotspot or graph" 2>&1 | tail -4
timeout 900 compute-sanitizer --tool racecheck --error-exitcode 9 python scripts/sanitize_smoke.py > gpurun_out/sanitize_racecheck.log 2>&1; echo "racecheck rc=$?"; tail -3 gpurun_out/sanitize_racecheck.log
timeout 600 compute-sanitizer --tool memcheck --error-exitcode 9 python scripts/sanitize_smoke.py > gpurun_out/sanitize_memcheck.log 2>&1; echo "memcheck rc=$?"; tail -3 gpurun_out/sanitize_memcheck.log
for ty in 64 128; do timeout 300 python bench.py --tile $ty --no-cpu-baseline --no-e2e > gpurun_out/bench_hot_ty$ty.log 2>&1; tail -c 330 gpurun_out/bench_hot_ty$ty.log | head -c 200; echo; done
timeout 400 ncu --set full --clock-control none --import-source on -k regex:hotspot -s 10 -c 1 -o gpurun_out/prof_hotspot_tma3d python bench.py --steps 1 --warmup 1 --iters 10 --no-e2e --no-cpu-baseline > /dev/null 2>&1
