timeout 900 python -m pytest tests/test_gpu_tpcc.py tests/test_gpu_small.py tests/test_gpu_carry.py tests/test_gpu_pipeline.py tests/test_gpu_multirank.py -x -q 2>&1 | tail -2
timeout 600 python bench.py --no-cpu-baseline > gpurun_out/bench_compact.json 2> gpurun_out/bench_compact.err
python -c "
import json; d=json.load(open('gpurun_out/bench_compact.json')); print(d['ms_per_step'], d['value'], d['e2e'], d['closed_loop_e2e']['value'], d['closed_loop_e2e']['h2d_bytes_per_step'])"
