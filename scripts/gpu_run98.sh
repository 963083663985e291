# repeatability: the GPU suite three times on one box (bit-identity assertions everywhere: a race would show)
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || tail -5 gpurun_out/build.log
for i in 1 2 3; do
timeout 1500 python -m pytest tests -m gpu -q -p no:randomly > gpurun_out/pytest_gpu_rep$i.log 2>&1; echo "run $i: $(tail -1 gpurun_out/pytest_gpu_rep$i.log)"
done
