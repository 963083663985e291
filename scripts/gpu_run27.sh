python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || true
OMP_NUM_THREADS=1 timeout 300 python -m torch.distributed.run --nnodes=1 --nproc-per-node=2 --master-addr=127.0.0.1 --master-port=29533 tests/spmd_ipc_worker.py /tmp/rep.json > gpurun_out/ipc2.log 2>&1; echo rc=$?
grep -v "^\s*$" gpurun_out/ipc2.log | grep -v "Setting OMP\|\*\*\*\*" | head -40
