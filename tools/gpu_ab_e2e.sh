timeout 900 python -m pytest tests/test_gpu_carry.py tests/test_gpu_tpcc.py tests/test_gpu_small.py -x -q 2>&1 | tail -1
for rep in 1 2; do for d in . _vhead; do
  (cd $d && timeout 600 python bench.py --no-cpu-baseline 2>/dev/null | python -c "
import json,sys; d=json.loads(sys.stdin.read()); e=d['e2e']; c=d['closed_loop_e2e']; print('%-7s e2e %.4f ms/step %.4g txn/s  closed-loop e2e %.4f ms/step %.4g  device %.4f' % ('$d', e['ms_per_step'], e['value'], c['ms_per_step'], c['value'], d['ms_per_step']))")
done; done
