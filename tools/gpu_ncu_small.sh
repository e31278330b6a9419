mkdir -p gpurun_out
export LTPG_NO_CLOCKS=1
timeout 600 /usr/local/cuda/bin/ncu --set full --clock-control none --import-source on -k regex:k_tpcc_small -s 4 -c 1 -f -o gpurun_out/full_small_c2 \
  python bench.py --workload tpcc_c2 --steps 2 --warmup 3 --no-cpu-baseline --no-e2e --no-closed-loop > gpurun_out/full_small_c2.log 2>&1
echo ncu rc=$?
