export LTPG_NO_CLOCKS=1
mkdir -p gpurun_out
/usr/local/cuda/bin/ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_e2e.csv \
  python bench.py --steps 2 --warmup 3 --no-cpu-baseline > gpurun_out/launch_e2e.log 2>&1
echo rc=$?
