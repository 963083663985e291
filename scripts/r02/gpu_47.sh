# round 2, call 47: per-kernel device times of C2 at P = 2 virtual partitions, pulled vs pushed halo
# (ncu launch lists; each command first run plainly)
for mode in pull push; do
  extra=""; [ $mode = push ] && extra="--push"
  python bench.py --workload hotspot2d --parts 2 --steps 2 --warmup 3 --no-e2e --no-cpu-baseline --no-e3 $extra > gpurun_out/r02_47_plain_$mode.log 2>&1 &&
  timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/r02_47_launches_$mode.csv python bench.py --workload hotspot2d --parts 2 --steps 2 --warmup 3 --no-e2e --no-cpu-baseline --no-e3 $extra > /dev/null 2>&1
  echo "== $mode"; python scripts/launch_summary.py gpurun_out/r02_47_launches_$mode.csv "bench --parts 2 $extra" | head -8
done
