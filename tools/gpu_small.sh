# TPC-C single-launch path: parity tests, stage timestamps (diagnostic build _vts), bench lines
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_small.py -x -q > gpurun_out/small_tests.log 2>&1; echo small tests rc=$?
tail -3 gpurun_out/small_tests.log
if [ -d _vts ]; then (cd _vts; for w in tpcc_c2 tpcc_c2_opt; do
  timeout 300 python bench.py --workload $w --steps 4 --warmup 3 --no-cpu-baseline --no-e2e --no-closed-loop 2>&1 | grep k_tpcc_small | tail -2
done); fi
for w in tpcc_c2 tpcc_c2_opt ycsb_c1; do
  timeout 300 python bench.py --workload $w --no-cpu-baseline > gpurun_out/bench_$w.json 2> gpurun_out/bench_$w.err
done
python - <<'P'
import json
for f in ["tpcc_c2", "tpcc_c2_opt", "ycsb_c1"]:
    try:
        d = json.load(open("gpurun_out/bench_%s.json" % f)); print(f, d["ms_per_step"], d["value"], d.get("e2e", {}).get("ms_per_step"), d.get("gpu_launches"))
    except Exception as e: print(f, "ERR", e)
P
