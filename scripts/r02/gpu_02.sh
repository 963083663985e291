# round 2, call 2: access-recording build + poison test
python -m paper_conf_icppw_matzdf20_b200.build --trace > gpurun_out/r02_02_build.log 2>&1 || tail -20 gpurun_out/r02_02_build.log
PK_TRACE_ACCESS=1 timeout 600 python tests/trace_worker.py > gpurun_out/r02_02_trace.jsonl 2> gpurun_out/r02_02_trace.err; echo "worker rc $?"
tail -5 gpurun_out/r02_02_trace.err
python -c "import json;[print(d[\"case\"],d[\"P\"],len(d[\"write_mismatch\"]),d[\"read_outside\"][:2],d[\"overfetch_words\"],d[\"declared_unfetched_words\"],d[\"stray\"]) for d in map(json.loads,open(\"gpurun_out/r02_02_trace.jsonl\"))]"
timeout 900 python -m pytest tests/test_gpu_access.py tests/test_gpu_trace.py -q -x > gpurun_out/r02_02_pytest.log 2>&1; tail -30 gpurun_out/r02_02_pytest.log
