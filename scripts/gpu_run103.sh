# final check after the heat3d_tb2 index change: memcheck + synccheck over every builtin kernel, smoke, default bench
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || tail -5 gpurun_out/build.log
for tool in memcheck synccheck; do
timeout 900 compute-sanitizer --tool $tool python scripts/sanitize_smoke.py > gpurun_out/sanitize_$tool.log 2>&1; echo "$tool rc=$?"; tail -2 gpurun_out/sanitize_$tool.log
done
python -c "import __graft_entry__ as g; g.smoke(); print('smoke ok')" > gpurun_out/smoke.log 2>&1; tail -2 gpurun_out/smoke.log
timeout 600 python bench.py > gpurun_out/bench_default.json 2> gpurun_out/bench_default.err; tail -c 300 gpurun_out/bench_default.json
