(cd _volrb && timeout 900 python -m pytest tests/test_gpu_tpcc.py tests/test_gpu_tpcc_pins.py -x -q 2>&1 | tail -1)
bash tools/ab.sh .,_volrb tpcc_c4 tpcc_c5 tpcc_c4_delayed
