# e2e pipeline depth: 2 vs 3 contexts (C2, C3, C4)
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || tail -5 gpurun_out/build.log
for w in hotspot2d heat3d sgemm; do for n in 2 3; do
PK_E2E_CONTEXTS=$n timeout 600 python bench.py --workload $w --steps 2 --warmup 3 --no-cpu-baseline > /tmp/b.log 2>&1; tail -1 /tmp/b.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$w ctx=$n', round(d['value'],1), round(d['e2e']['value'],1), d['e2e']['timing'][:90])" || tail -3 /tmp/b.log
done; done
