#!/bin/bash
# Bench lines of the main workloads into gpurun_out/bench_<tag>_<workload>.json (run on the GPU box)
TAG=${1:-r01}
mkdir -p gpurun_out
python bench.py > gpurun_out/bench_${TAG}_default.json 2> gpurun_out/bench_${TAG}_default.err
python bench.py --workload ycsb_c3 > gpurun_out/bench_${TAG}_ycsb_c3.json 2> gpurun_out/bench_${TAG}_ycsb_c3.err
for w in tpcc_c2 ycsb_c1 tpcc_c4_delayed tpcc_c4_opt tpcc_c5 ycsb_a ycsb_e; do
  python bench.py --workload $w --no-cpu-baseline > gpurun_out/bench_${TAG}_$w.json 2> gpurun_out/bench_${TAG}_$w.err
done
python bench.py --impl reference --steps 3 --warmup 3 > gpurun_out/bench_${TAG}_reference.json 2> gpurun_out/bench_${TAG}_reference.err
