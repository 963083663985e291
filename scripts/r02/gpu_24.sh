# round 2, call 24: heat3d_tb2 planes per block vs waves (9 x 64 x ceil(1024/ZC) blocks on 444 CTA slots)
run() {
  timeout 300 python bench.py --workload heat3d --tile $1 --steps 5 --no-e2e --no-cpu-baseline --no-e3 > /tmp/b.json 2> /tmp/b.err
  tail -1 /tmp/b.json | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('ZC', $1, round(d['value'],1), 'frac', round(d['roofline']['frac'],4), round(d['kernel_ms_avg'],4), d['clocks']['sm_mhz'], d['clocks']['reasons'])" || tail -3 /tmp/b.err
}
for z in 64 79 103 128 64 103; do run $z; done
timeout 600 python -m pytest tests/test_gpu_parity.py -q -x -k "aliased" 2>&1 | tail -1
