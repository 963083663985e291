# round 2, call 74: ncu of the C1 default kernel (jacobi2d_tb, K = 5): launch list of the bench + one full capture
python bench.py --workload jacobi2d --steps 2 --warmup 3 --no-e2e --no-cpu-baseline --no-e3 > gpurun_out/r02_74_plain.log 2>&1 &&
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/r02_74_launches.csv python bench.py --workload jacobi2d --steps 2 --warmup 3 --no-e2e --no-cpu-baseline --no-e3 > /dev/null 2>&1
python scripts/launch_summary.py gpurun_out/r02_74_launches.csv "bench --workload jacobi2d" | head -5
mkdir -p gpurun_out/r02_74
timeout 600 ncu --set full --clock-control none --import-source on -k regex:jacobi2d_tb -s 10 -c 1 -o gpurun_out/r02_74/jtb5 python bench.py --workload jacobi2d --steps 2 --warmup 3 --no-e2e --no-cpu-baseline --no-e3 > /dev/null 2>&1; echo ncu rc $?
