# compute-sanitizer over every builtin kernel incl. tb2/tbK (K = 4, 8), heat3d_tb2, async copies and push
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || tail -5 gpurun_out/build.log
for tool in memcheck racecheck synccheck; do
timeout 900 compute-sanitizer --tool $tool python scripts/sanitize_smoke.py > gpurun_out/sanitize_$tool.log 2>&1; echo "$tool rc=$?"; tail -2 gpurun_out/sanitize_$tool.log
done
