b() { timeout 300 python bench.py --no-e2e --no-cpu-baseline --steps 10 --warmup 3 --variant hotspot2d_tbk --sweeps 4 $1 > gpurun_out/b.log 2>&1; tail -1 gpurun_out/b.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$2 $1', round(d['value'],1), round(d['roofline']['frac'],3), round(d['kernel_ms_avg'],4))" || tail -3 gpurun_out/b.log; }
for v in "-DPK_TBK_MINB=4 -DPK_TBK_NS=8" "-DPK_TBK_NS=8" "-DPK_TBK_NS=16"; do
PK_NVCC_FLAGS="$v" python -c "from paper_conf_icppw_matzdf20_b200 import build; build.build(force=True)" > /dev/null 2>&1
b "--tile 112" "$v"
done
for TY in 80 96 144 160 192; do b "--tile $TY" "NS16"; done
