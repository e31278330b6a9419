(cd _vts
for w in ycsb_c1 tpcc_c2; do
timeout 300 python bench.py --workload $w --steps 4 --warmup 3 --no-cpu-baseline --no-e2e --no-closed-loop 2>&1 | grep 'k_ops_small\|k_tpcc_small' | tail -3
done)
