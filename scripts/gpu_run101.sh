# heat3d_tb2 with 32-bit row/plane indices: GPU suite, heat bench line, ncu full summary + launch list
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || tail -5 gpurun_out/build.log
timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1; tail -1 gpurun_out/pytest_gpu.log
timeout 300 python bench.py --workload heat3d > gpurun_out/bench_heat3d.json 2> gpurun_out/bench_heat3d.err; tail -c 400 gpurun_out/bench_heat3d.json
timeout 600 ncu --set full --clock-control none --import-source on -k regex:heat3d_tb2 -s 3 -c 1 -o gpurun_out/prof_heat_tb2_i32 python bench.py --workload heat3d --steps 1 --warmup 1 --iters 10 --no-e2e --no-cpu-baseline > /dev/null 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/launches_heat3d_i32.csv python bench.py --workload heat3d --steps 2 --warmup 1 --no-e2e --no-cpu-baseline > /dev/null 2>&1
ls gpurun_out
