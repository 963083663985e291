# round 2, call 43: GPU suite after the transfer-pass restructure (waits for every destination before
# any copy) + A/B against the previous build on virtual-partition runs where transfers matter
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/r02_43_build.log 2>&1 || tail -5 gpurun_out/r02_43_build.log
timeout 1800 python -m pytest tests -m gpu -q -x > gpurun_out/r02_43_pytest_gpu.log 2>&1; echo "gpu suite: $(tail -1 gpurun_out/r02_43_pytest_gpu.log)"
: > gpurun_out/r02_43_ab.txt
for rep in 1 2; do
for lib in old new; do
  if [ $lib = old ]; then export PK_LIB_OVERRIDE=$PWD/scratch/libpk_before_passes.so; else unset PK_LIB_OVERRIDE; fi
  for spec in "jacobi2d 2" "jacobi2d 4" "jacobi2d 8" "hotspot2d 8" "heat3d 8" "nbody 8"; do
    set -- $spec; w=$1; P=$2
    st=10; [ $w = nbody ] && st=2
    timeout 600 python bench.py --workload $w --parts $P --steps $st --warmup 3 --no-e2e --no-cpu-baseline --no-e3 > /tmp/b.log 2>&1
    tail -1 /tmp/b.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); t=d['transfers']; print('$lib $w P=$P', round(d['value'],2), d['unit'], 'ms/step', round(d['ms_per_step'],4), 'moved', t['moved_bytes'], 'min', t['analytic_min_bytes'])" >> gpurun_out/r02_43_ab.txt 2>&1 || tail -3 /tmp/b.log >> gpurun_out/r02_43_ab.txt
  done
done
done
unset PK_LIB_OVERRIDE
cat gpurun_out/r02_43_ab.txt
