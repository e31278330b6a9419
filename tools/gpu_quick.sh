# quick GPU check: TPC-C parity files + default / c5 / c2 bench lines (run on the GPU box)
mkdir -p gpurun_out
timeout 1200 python -m pytest tests/test_gpu_tpcc.py tests/test_gpu_small.py tests/test_gpu_partitions.py tests/test_gpu_multirank.py tests/test_gpu_pipeline.py -x -q > gpurun_out/quick_tests.log 2>&1; echo tests rc=$?
tail -2 gpurun_out/quick_tests.log
for w in default tpcc_c5 tpcc_c2 tpcc_c4_delayed; do
  if [ $w = default ]; then a=""; else a="--workload $w --no-cpu-baseline"; fi
  timeout 600 python bench.py $a > gpurun_out/bench_$w.json 2> gpurun_out/bench_$w.err
done
python - <<'P'
import json
for f in ["default", "tpcc_c5", "tpcc_c2", "tpcc_c4_delayed"]:
    try:
        d = json.load(open("gpurun_out/bench_%s.json" % f)); s = d["stage_ms_mean"]
        print(f, "%.4f" % d["ms_per_step"], "%.4g" % d["value"], " ".join("%s=%.4f" % (k[3:], v) for k, v in s.items()))
    except Exception as e: print(f, "ERR", e)
P
