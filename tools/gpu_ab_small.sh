timeout 900 python -m pytest tests/test_gpu_small.py tests/test_gpu_ops.py tests/test_gpu_ycsb_suite.py -x -q 2>&1 | tail -1
bash tools/ab.sh .,_vhead ycsb_c1 ycsb_c1 tpcc_c2
