timeout 900 python -m pytest tests/test_gpu_tpcc.py tests/test_gpu_small.py tests/test_gpu_partitions.py tests/test_gpu_pipeline.py tests/test_gpu_carry.py -x -q 2>&1 | tail -2
bash tools/ab.sh .,_vx1 tpcc_c4 tpcc_c5
