#!/bin/bash
# Profile one bench workload on the GPU box (run under gpurun, one GPU):
#   tools/profile.sh WORKLOAD KERNEL_REGEX SKIP COUNT
# 1) launch list: every kernel of `bench.py --steps 2 --warmup 3` (cold-cache, serialised)
# 2) `ncu --set full` of COUNT launches matching KERNEL_REGEX after skipping SKIP of them
# Outputs land in gpurun_out/ (summarise with tools/ncu_summary.py, commit under profiles/).
W=$1; K=$2; SKIP=${3:-0}; CNT=${4:-8}
NCU=/usr/local/cuda/bin/ncu
mkdir -p gpurun_out
export LTPG_NO_CLOCKS=1
$NCU --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_$W.csv \
  python bench.py --workload $W --steps 2 --warmup 3 --no-cpu-baseline --no-closed-loop > gpurun_out/launch_$W.log 2>&1
echo "launch list rc=$?"
$NCU --set full --clock-control none --import-source on -k "regex:$K" -s $SKIP -c $CNT -f -o gpurun_out/full_$W \
  python bench.py --workload $W --steps 2 --warmup 3 --no-cpu-baseline --no-e2e --no-closed-loop > gpurun_out/full_$W.log 2>&1
echo "full rc=$?"
