# e2e diagnosis: pipelined vs blocking, per-step enqueue times
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || tail -5 gpurun_out/build.log
for env in "PK_E2E_TRACE=1" "PK_E2E_TRACE=1 PK_E2E_BLOCKING=1"; do
env $env timeout 600 python bench.py --steps 2 --warmup 3 --no-cpu-baseline > /tmp/b.log 2>/tmp/e.log; grep "e2e step" /tmp/e.log | tr '\n' ' '; echo
tail -1 /tmp/b.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('[$env]', d['e2e']['value'], d['value'])"
done
