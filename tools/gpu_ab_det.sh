timeout 900 python -m pytest tests/test_gpu_tpcc.py tests/test_gpu_small.py tests/test_gpu_reorder.py tests/test_gpu_buckets.py tests/test_gpu_ops.py -x -q 2>&1 | tail -2
bash tools/ab.sh .,_vhead tpcc_c4 tpcc_c4_opt ycsb_c3
