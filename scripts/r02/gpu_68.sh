# round 2, call 68: ncu of jacobi2d_tb (K = 10) at P = 1
mkdir -p gpurun_out/r02_68
python bench.py --workload jacobi2d --variant jacobi2d_tb --steps 2 --warmup 3 --no-e2e --no-cpu-baseline --no-e3 > gpurun_out/r02_68_plain.log 2>&1 &&
timeout 600 ncu --set full --clock-control none --import-source on -k regex:jacobi2d_tb -s 5 -c 1 -o gpurun_out/r02_68/jtb python bench.py --workload jacobi2d --variant jacobi2d_tb --steps 2 --warmup 3 --no-e2e --no-cpu-baseline --no-e3 > /dev/null 2>&1; echo ncu rc $?
