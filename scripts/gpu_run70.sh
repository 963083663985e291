python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || tail -5 gpurun_out/build.log
timeout 900 ncu --set full --clock-control none --import-source on -k regex:nbody_partial -s 3 -c 1 -o gpurun_out/prof_nbody4 python bench.py --workload nbody --steps 1 --warmup 3 --iters 1 --no-e2e --no-cpu-baseline > gpurun_out/prof_nbody4.log 2>&1
tail -2 gpurun_out/prof_nbody4.log
