timeout 900 python -m pytest tests/test_gpu_small.py tests/test_gpu_ops.py tests/test_gpu_ycsb_suite.py tests/test_gpu_reorder.py tests/test_gpu_graph.py tests/test_gpu_pipeline.py -x -q 2>&1 | tail -2
bash tools/ab.sh .,_vkg ycsb_c1 ycsb_c1
