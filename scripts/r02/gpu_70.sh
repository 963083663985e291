# round 2, call 70: jacobi2d_tb sweeps per launch K = 2..10 at P = 1 and P = 2, sweep loop unrolled or not
run() {
  timeout 300 python bench.py --workload jacobi2d --no-e2e --no-cpu-baseline --no-e3 $2 > /tmp/b.json 2> /tmp/b.err
  tail -1 /tmp/b.json | python -c "import json,sys; d=json.loads(sys.stdin.read()); t=d['transfers']; print('$1', round(d['value'],1), 'us/step', round(1e3*d['ms_per_step'],1), 'launches', d['gpu_launches'], 'moved', t['moved_bytes'])" || tail -3 /tmp/b.err
}
for U in 1 0; do
  PK_NVCC_FLAGS="-DPK_JTB_SUNROLL=$U" python -m paper_conf_icppw_matzdf20_b200.build > /dev/null 2>&1 || echo BUILD FAIL
  for P in 1 2; do
    run "unroll=$U jacobi2d      P=$P" "--parts $P"
    for k in 2 3 4 5 6 8 10; do
      run "unroll=$U tb K=$k        P=$P" "--parts $P --variant jacobi2d_tb --sweeps $k"
    done
  done
done
python -m paper_conf_icppw_matzdf20_b200.build > /dev/null 2>&1
