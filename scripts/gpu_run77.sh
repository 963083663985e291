# SPMD bench path (the driver's --gpus N launch) with 2 ranks time-slicing the one GPU: functional check
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || tail -5 gpurun_out/build.log
for w in hotspot2d heat3d; do
timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29611 bench.py --gpus 2 --workload $w --steps 3 --warmup 3 > gpurun_out/spmd2_$w.log 2>&1; echo "rc=$?"
tail -1 gpurun_out/spmd2_$w.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$w', d['n_gpus'], round(d['value'],1), d['transfers'], d['e2e']['value'], d['config']['process_model'][:40])" || tail -5 gpurun_out/spmd2_$w.log
done
timeout 300 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29612 bench.py --gpus 2 --impl reference --steps 2 --warmup 1 2>&1 | tail -1 | cut -c1-200
