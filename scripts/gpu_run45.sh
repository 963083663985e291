r() { (cd $1 && timeout 600 python bench.py $2 --steps 10 --warmup 3 --no-e2e --no-cpu-baseline > /tmp/b.log 2>&1; tail -1 /tmp/b.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$1 $2', round(d['value'],1), round(d['roofline']['frac'],3), d['clocks']['sm_mhz'], d['clocks']['power_w_max'])"); }
for i in 1 2; do
r ab_old ""; r . ""; r ab_old "--workload heat3d"; r . "--workload heat3d"
done
