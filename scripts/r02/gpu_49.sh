# round 2, call 49: compute-sanitizer memcheck over every builtin after the push post-pass and the
# three-pass transfer ordering (one sanitizer tool per call)
python scripts/sanitize_smoke.py > gpurun_out/r02_49_plain.log 2>&1 && \
timeout 1200 compute-sanitizer --tool memcheck --error-exitcode 9 python scripts/sanitize_smoke.py > gpurun_out/r02_49_memcheck.log 2>&1; echo "memcheck rc=$?"; grep -E "SUMMARY|sanitize smoke done" gpurun_out/r02_49_memcheck.log | tail -3
