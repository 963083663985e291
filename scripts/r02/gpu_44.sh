# round 2, call 44: C1 at P = 2 with the fused halo push vs pulled copies; ncu --set full of the
# default bench kernel (C2 hotspot2d_tbk, K = 4) with the round-2 build
: > gpurun_out/r02_44_c1.txt
for rep in 1 2 3; do
  for mode in pull push; do
    extra=""; [ $mode = push ] && extra="--push"
    timeout 300 python bench.py --workload jacobi2d --parts 2 --steps 10 --warmup 3 --no-e2e --no-cpu-baseline --no-e3 $extra > /tmp/b.log 2>&1
    tail -1 /tmp/b.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); t=d['transfers']; print('$mode P=2', round(d['value'],2), d['unit'], 'ms/step', round(d['ms_per_step'],4), 'moved', t['moved_bytes'], 'pushed', t['pushed_bytes'], 'min', t['analytic_min_bytes'])" >> gpurun_out/r02_44_c1.txt 2>&1 || tail -3 /tmp/b.log >> gpurun_out/r02_44_c1.txt
  done
done
cat gpurun_out/r02_44_c1.txt
mkdir -p gpurun_out/r02_44
python bench.py --steps 2 --warmup 3 --no-e2e --no-cpu-baseline --no-e3 > gpurun_out/r02_44_plain.log 2>&1 &&
timeout 900 ncu --set full --clock-control none --import-source on -k regex:hotspot2d_tbk -s 30 -c 1 -o gpurun_out/r02_44/c2_tbk python bench.py --steps 2 --warmup 3 --no-e2e --no-cpu-baseline --no-e3 > gpurun_out/r02_44_ncu.log 2>&1; echo ncu rc $?
