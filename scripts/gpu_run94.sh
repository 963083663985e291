python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || tail -5 gpurun_out/build.log
timeout 600 ncu --set full --clock-control none --import-source on -k regex:tbk -s 5 -c 1 -o gpurun_out/prof_tbk_final python bench.py --steps 1 --warmup 1 --iters 24 --no-e2e --no-cpu-baseline > gpurun_out/prof_tbk_final.log 2>&1
tail -1 gpurun_out/prof_tbk_final.log
