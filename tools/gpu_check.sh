# HEAD check: full GPU suite, smoke(), default bench line
mkdir -p gpurun_out
timeout 1800 python -m pytest tests -m gpu -x -q > gpurun_out/gputest_head.log 2>&1; echo gputest rc=$?
tail -2 gpurun_out/gputest_head.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -2
timeout 600 python bench.py > gpurun_out/bench_head_default.json 2> gpurun_out/bench_head_default.err; echo bench rc=$?
python tools/design_table.py head_default gpurun_out 2>/dev/null | tail -1
python -c "
import json; d=json.load(open('gpurun_out/bench_head_default.json')); print(d['ms_per_step'], d['value'], d['e2e']['value'], d['e2e']['ms_per_step'], d['closed_loop_e2e']['value'], d['roofline']['frac'], d['clocks']['reasons'], d['gpu_launches'])"
