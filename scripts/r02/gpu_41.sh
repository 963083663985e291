# round 2, call 41: compute-sanitizer over every builtin incl. C1 launch sequences with programmatic
# dependent launch and the heat3d_tb2 exchange buffer
python -m paper_conf_icppw_matzdf20_b200.build > /dev/null 2>&1 || echo BUILD FAIL
for tool in memcheck synccheck racecheck; do
  timeout 1200 compute-sanitizer --tool $tool --error-exitcode 9 python scripts/sanitize_smoke.py > gpurun_out/r02_41_$tool.log 2>&1; echo "$tool rc=$?"; grep -E "SUMMARY|sanitize smoke done" gpurun_out/r02_41_$tool.log | tail -3
done
