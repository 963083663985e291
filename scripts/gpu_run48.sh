python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || true
timeout 1500 python -m pytest tests -m gpu -q > gpurun_out/pytest_gpu.log 2>&1; tail -2 gpurun_out/pytest_gpu.log
OMP_NUM_THREADS=1 timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node=2 --master-addr=127.0.0.1 --master-port=29561 bench.py --gpus 2 --steps 3 --warmup 3 > gpurun_out/spmd2.log 2>&1; echo rc=$?; tail -1 gpurun_out/spmd2.log | cut -c1-300
OMP_NUM_THREADS=1 timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node=2 --master-addr=127.0.0.1 --master-port=29562 bench.py --impl reference --gpus 2 --steps 2 --warmup 1 > gpurun_out/spmd2ref.log 2>&1; echo rc=$?; tail -1 gpurun_out/spmd2ref.log | cut -c1-200
