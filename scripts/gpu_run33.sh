python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || true
timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -q -x -k "tbk" 2>&1 | tail -3
b() { timeout 300 python bench.py --no-e2e --no-cpu-baseline --steps 10 --warmup 3 --variant hotspot2d_tbk --sweeps 4 $1 > gpurun_out/b.log 2>&1; tail -1 gpurun_out/b.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$2 $1', round(d['value'],1), round(d['roofline']['frac'],3), round(d['kernel_ms_avg'],4))" || tail -3 gpurun_out/b.log; }
b "" minb1
b "--tile 256" minb1
for m in 2; do
PK_NVCC_FLAGS="-DPK_TBK_MINB=$m" python -c "from paper_conf_icppw_matzdf20_b200 import build; build.build(force=True)" > /dev/null 2>&1
b "" minb$m
b "--tile 256" minb$m
done
