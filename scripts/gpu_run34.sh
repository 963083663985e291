python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || true
ncu --set full --import-source on --clock-control none -k regex:k_hotspot2d_tbk -c 1 -s 5 -o gpurun_out/tbk4b python bench.py --no-e2e --no-cpu-baseline --steps 1 --warmup 3 --variant hotspot2d_tbk --sweeps 4 > /dev/null 2>&1
ls -la gpurun_out/tbk4b.ncu-rep
