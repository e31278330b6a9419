# full GPU suite + default bench line (run on the GPU box)
mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/gputest.log 2>&1; echo gputest rc=$?
tail -3 gpurun_out/gputest.log
timeout 600 python bench.py > gpurun_out/bench_default.json 2> gpurun_out/bench_default.err; echo bench rc=$?
python - <<'P'
import json
d = json.load(open("gpurun_out/bench_default.json"))
print(d["ms_per_step"], d["value"], d["stage_ms_mean"], d["e2e"]["value"], d["roofline"]["frac"])
P
