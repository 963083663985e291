# round 2, call 26: shorter dependency chains in the stencil updates (tree-shaped sums) vs round 1's sequential sums
KD=paper_conf_icppw_matzdf20_b200/csrc/kernels
run() {
  timeout 300 python bench.py --workload $1 --steps 10 --no-e2e --no-cpu-baseline --no-e3 > /tmp/b.json 2> /tmp/b.err
  tail -1 /tmp/b.json | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$1 $2', round(d['value'],1), 'frac', round(d['roofline']['frac'],4), 'kms', round(d['kernel_ms_avg'],4), d['clocks']['sm_mhz'], d['clocks']['reasons'])" || tail -3 /tmp/b.err
}
for r in 1 2 3; do
  for v in r1 tree; do
    cp scratch/hotspot_tbk_$v.cu $KD/hotspot_tbk.cu; cp scratch/heat_tb_$v.cu $KD/heat_tb.cu
    python -m paper_conf_icppw_matzdf20_b200.build > /dev/null 2>&1 || echo BUILD FAIL $v
    run hotspot2d $v; run heat3d $v
  done
done
timeout 600 python -m pytest tests/test_gpu_parity.py tests/test_gpu_fullsize.py -q -x -k "hotspot or heat or c2 or c3" > gpurun_out/r02_26_pytest.log 2>&1; echo "tree parity: $(tail -1 gpurun_out/r02_26_pytest.log)"
