# round 2, call 3: GPU suite with the new timing / E3 / direct launch; bench lines; peak probes
python -m paper_conf_icppw_matzdf20_b200.build > /dev/null 2>&1 || echo BUILD FAILED
timeout 1500 python -m pytest tests -m gpu -q -x > gpurun_out/r02_03_pytest.log 2>&1; echo "gpu suite: $(tail -1 gpurun_out/r02_03_pytest.log)"
grep -E "FAILED|Error" gpurun_out/r02_03_pytest.log | head -20
timeout 300 python scripts/probe_peaks.py > gpurun_out/r02_03_peaks.json 2>&1; tail -c 1500 gpurun_out/r02_03_peaks.json
for wl in hotspot2d sgemm; do
  timeout 600 python bench.py --workload $wl > gpurun_out/r02_03_bench_$wl.json 2> gpurun_out/r02_03_bench_$wl.err
  tail -1 gpurun_out/r02_03_bench_$wl.json | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$wl', round(d['value'],1), d['unit'], d['roofline']['frac'], d['roofline']['peak'], d['kernel_timing'][:80], d.get('e3_single_gpu_slowdown'), d['host_us_per_launch'], d['host_cpu_us_per_launch'], d['host_us_per_launch_timed_region'], d['clocks'])" || tail -5 gpurun_out/r02_03_bench_$wl.err
done
timeout 600 python bench.py --workload hotspot2d --parts 4 --abg --no-e2e --no-cpu-baseline --steps 5 > gpurun_out/r02_03_bench_abg.json 2> gpurun_out/r02_03_bench_abg.err
tail -1 gpurun_out/r02_03_bench_abg.json | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('abg', round(d['value'],1), d['overhead'], d['transfers'])" || tail -5 gpurun_out/r02_03_bench_abg.err
timeout 600 python bench.py --workload sgemm --parts 4 --no-e2e --no-cpu-baseline --steps 4 > gpurun_out/r02_03_bench_sgemm4.json 2> gpurun_out/r02_03_bench_sgemm4.err
tail -1 gpurun_out/r02_03_bench_sgemm4.json | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('sgemm P4', round(d['value'],1), d['roofline']['frac'], d['transfers'], d['kernel_timing'][:100])" || tail -5 gpurun_out/r02_03_bench_sgemm4.err
