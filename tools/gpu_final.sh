# round-end evidence at HEAD: full GPU suite, every workload's bench line, ncu of tpcc_c4's phase
# kernels and of the single-launch kernels (tpcc_c2, ycsb_c1)
mkdir -p gpurun_out
timeout 1800 python -m pytest tests -m gpu -x -q > gpurun_out/gputest_final.log 2>&1; echo gputest rc=$?
tail -2 gpurun_out/gputest_final.log
bash tools/gpu_sweep.sh ${1:-r02f}
