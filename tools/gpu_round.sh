set -x
python -m pytest tests -m gpu -x -q > gpurun_out/gputest.log 2>&1; echo gputest rc=$?
tail -3 gpurun_out/gputest.log
python bench.py > gpurun_out/bench_r02b_default.json 2> gpurun_out/bench_r02b_default.err; echo bench rc=$?
python bench.py --workload tpcc_c2 --no-cpu-baseline > gpurun_out/bench_r02b_tpcc_c2.json 2> gpurun_out/bench_r02b_tpcc_c2.err
python bench.py --workload ycsb_c1 --no-cpu-baseline > gpurun_out/bench_r02b_ycsb_c1.json 2> gpurun_out/bench_r02b_ycsb_c1.err
bash tools/profile.sh tpcc_c4 'k_tpcc|k_no_|k_sl_|k_finalize|k_publish|k_batch' 14 16
bash tools/profile.sh tpcc_c2 'k_tpcc|k_no_|k_sl_|k_finalize|k_publish|k_batch' 14 16
