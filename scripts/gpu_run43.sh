python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || true
timeout 600 python bench.py --impl reference --steps 2 --warmup 1 > gpurun_out/ref.log 2>&1; tail -1 gpurun_out/ref.log
for wl in heat3d sgemm nbody jacobi2d; do
timeout 600 python bench.py --workload $wl --steps 5 --warmup 3 > gpurun_out/bench_$wl.log 2>&1; tail -1 gpurun_out/bench_$wl.log | cut -c1-400
done
ncu --set full --import-source on --clock-control none -k regex:k_sgemm_tf32x3 -c 1 -s 1 -o gpurun_out/sgemm_chunked python bench.py --workload sgemm --no-e2e --no-cpu-baseline --steps 1 --warmup 3 > /dev/null 2>&1
ls gpurun_out
