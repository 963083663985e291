# round 2, call 45: fused halo push vs pulled copies at P = 2/4/8 virtual partitions (C2, C3), and the
# SPMD peer-memory path with push (2 ranks sharing the GPU: functional only)
: > gpurun_out/r02_45_push.txt
for rep in 1 2; do
  for spec in "hotspot2d 2" "hotspot2d 8" "heat3d 2" "heat3d 8"; do
    set -- $spec; w=$1; P=$2
    for mode in pull push; do
      extra=""; [ $mode = push ] && extra="--push"
      timeout 600 python bench.py --workload $w --parts $P --steps 10 --warmup 3 --no-e2e --no-cpu-baseline --no-e3 $extra > /tmp/b.log 2>&1
      tail -1 /tmp/b.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); t=d['transfers']; print('$mode $w P=$P', round(d['value'],2), d['unit'], 'ms/step', round(d['ms_per_step'],4), 'moved', t['moved_bytes'], 'pushed', t['pushed_bytes'], 'min', t['analytic_min_bytes'], d['clocks']['sm_mhz'])" >> gpurun_out/r02_45_push.txt 2>&1 || tail -3 /tmp/b.log >> gpurun_out/r02_45_push.txt
    done
  done
done
cat gpurun_out/r02_45_push.txt
timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29545 bench.py --gpus 2 --steps 3 --warmup 3 --push --no-e2e > gpurun_out/r02_45_n2_push.json 2> gpurun_out/r02_45_n2_push.err; echo "n2 push rc $?"; tail -c 600 gpurun_out/r02_45_n2_push.json; echo
