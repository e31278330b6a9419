#!/bin/bash
# Bench lines of the main workloads into gpurun_out/bench_<tag>_<workload>.json (run on the GPU box)
TAG=${1:-r02}
mkdir -p gpurun_out
python bench.py > gpurun_out/bench_${TAG}_default.json 2> gpurun_out/bench_${TAG}_default.err
python bench.py --workload ycsb_c3 > gpurun_out/bench_${TAG}_ycsb_c3.json 2> gpurun_out/bench_${TAG}_ycsb_c3.err
for w in tpcc_c2 ycsb_c1 tpcc_c4_delayed tpcc_c4_opt tpcc_c5 ycsb_a ycsb_e ycsb_c3_4ops ycsb_c3_sparse tpcc_c2_opt; do
  python bench.py --workload $w --no-cpu-baseline > gpurun_out/bench_${TAG}_$w.json 2> gpurun_out/bench_${TAG}_$w.err
done
# multi-rank (ranks share the one GPU here: a functional check of the sharded path, not scaling)
for g in 2 4; do
  python bench.py --gpus $g --steps 5 > gpurun_out/bench_${TAG}_gpus$g.json 2> gpurun_out/bench_${TAG}_gpus$g.err
done
# NEXT-3 A/B: large-sized hash buckets (flag 32), with and without the mark filter (flag 2)
for f in 2 32 34; do
  for w in tpcc_c2 tpcc_c4; do
    python bench.py --workload $w --flags $f --no-cpu-baseline --no-e2e > gpurun_out/bench_${TAG}_${w}_flags$f.json 2> /dev/null
  done
done
python bench.py --impl reference > gpurun_out/bench_${TAG}_reference.json 2> gpurun_out/bench_${TAG}_reference.err
