#!/bin/bash
# compute-sanitizer memcheck / racecheck / synccheck over small runs (GPU box, one GPU):
#   tools/sanitize.sh  -> gpurun_out/sanitize_<tool>_<run>.txt
CS=/usr/local/cuda/bin/compute-sanitizer
mkdir -p gpurun_out
for tool in memcheck racecheck synccheck; do
  for run in ycsb_c1 tpcc_c2 ycsb_e carry; do
    timeout 900 $CS --tool $tool --print-limit 50 python tests/sanitize_run.py $run > gpurun_out/sanitize_${tool}_${run}.txt 2>&1
    echo "$tool $run rc=$?"; tail -2 gpurun_out/sanitize_${tool}_${run}.txt
  done
  for mr in multirank multirank_sharded; do
    timeout 900 $CS --tool $tool --print-limit 50 --target-processes all python -m torch.distributed.run --nnodes=1 \
      --nproc-per-node=2 --master-addr=127.0.0.1 --master-port=29533 tests/sanitize_run.py $mr \
      > gpurun_out/sanitize_${tool}_$mr.txt 2>&1
    echo "$tool $mr rc=$?"; tail -3 gpurun_out/sanitize_${tool}_$mr.txt
  done
done
