python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || true
s=$(date +%s); timeout 900 python bench.py > gpurun_out/bench_default.log 2>gpurun_out/bench_default.err; echo "bench default wall $(( $(date +%s) - s )) s"
tail -1 gpurun_out/bench_default.log > gpurun_out/bench_default.json
python -c "import json; d=json.load(open('gpurun_out/bench_default.json')); print(d['value'], d['roofline']['frac'], d['e2e']['value'], d['cpu_baseline'], d['clocks'])"
bash scripts/gpu_run72.sh
