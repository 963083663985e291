python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || true
timeout 900 python -m pytest tests/test_gpu_spmd_ipc.py -m gpu -q -x 2>&1 | tail -3
for N in 2 4; do
OMP_NUM_THREADS=1 timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node=$N --master-addr=127.0.0.1 --master-port=2954$N bench.py --gpus $N --steps 3 --warmup 3 --no-e2e > gpurun_out/bench_spmd$N.log 2>&1; echo rc=$?
tail -1 gpurun_out/bench_spmd$N.log | cut -c1-900
done
OMP_NUM_THREADS=1 timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node=2 --master-addr=127.0.0.1 --master-port=29561 bench.py --gpus 2 --steps 3 --warmup 3 > gpurun_out/bench_spmd2e.log 2>&1; echo rc=$?
tail -1 gpurun_out/bench_spmd2e.log | cut -c1-1500
