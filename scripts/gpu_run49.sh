python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || true
timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -q -x -k "tb2" 2>&1 | tail -3
r() { timeout 600 python bench.py $1 --steps 5 --warmup 3 --no-e2e --no-cpu-baseline > /tmp/b.log 2>&1; tail -1 /tmp/b.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$1 $2', round(d['value'],1), round(d['roofline']['frac'],3), round(d['kernel_ms_avg'],4))" || tail -3 /tmp/b.log; }
r "--workload heat3d --variant heat3d_tb2" minb1
r "--workload heat3d --variant heat3d_tb2 --tile 256" minb1
PK_NVCC_FLAGS="-DPK_HEATTB_MINB=2" python -c "from paper_conf_icppw_matzdf20_b200 import build; build.build(force=True)" > /dev/null 2>&1
r "--workload heat3d --variant heat3d_tb2" minb2
r "--workload heat3d" base
