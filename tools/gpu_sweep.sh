# round-2 sweep at HEAD: every workload's bench line + ncu of the tpcc_c4 phase kernels and of the
# single-launch kernels (tpcc_c2, ycsb_c1).  Outputs in gpurun_out/ (summarise into profiles/).
TAG=${1:-r02c}
bash tools/bench_all.sh $TAG
bash tools/profile.sh tpcc_c4 'k_tpcc|k_no_|k_sl_|k_finalize|k_publish|k_batch' 14 16
export LTPG_NO_CLOCKS=1
for w in tpcc_c2 ycsb_c1; do
  /usr/local/cuda/bin/ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_$w.csv \
    python bench.py --workload $w --steps 2 --warmup 3 --no-cpu-baseline --no-closed-loop > gpurun_out/launch_$w.log 2>&1
  /usr/local/cuda/bin/ncu --set full --clock-control none --import-source on -k regex:'k_tpcc_small|k_ops_small' -s 4 -c 1 -f -o gpurun_out/full_$w \
    python bench.py --workload $w --steps 2 --warmup 3 --no-cpu-baseline --no-e2e --no-closed-loop > gpurun_out/full_$w.log 2>&1
  echo ncu $w rc=$?
done
