# heat3d_tb2: one ncu --set full capture with source + stall reasons (where the 2-sweep kernel loses vs the ring alone)
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || tail -5 gpurun_out/build.log
timeout 600 ncu --set full --clock-control none --import-source on -k regex:heat3d_tb2 -s 3 -c 1 -o gpurun_out/prof_heat_tb2_r01b python bench.py --workload heat3d --steps 1 --warmup 1 --iters 10 --no-e2e --no-cpu-baseline > gpurun_out/prof_heat.log 2>&1
ls -la gpurun_out
