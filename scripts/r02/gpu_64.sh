# round 2, call 64: the GPU suite twice more on one box (repeatability of the bit-identity assertions with
# the final build)
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
for r in 1 2; do
  timeout 1800 python -m pytest tests -m gpu -q -p no:randomly > gpurun_out/r02_64_pytest_$r.log 2>&1; echo "run $r: $(tail -1 gpurun_out/r02_64_pytest_$r.log)"
done
