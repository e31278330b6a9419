#!/bin/bash
# A/B on one GPU box: tools/ab.sh DIR_A DIR_B WORKLOAD... (each a repo checkout with built .so)
A=$1; B=$2; shift 2
for w in "$@"; do
  for rep in 1 2; do
    for d in $A $B; do
      (cd $d && python bench.py --workload $w --no-cpu-baseline --no-e2e 2>/dev/null | tail -1 | python -c "
import json,sys; d=json.loads(sys.stdin.read()); s=d['stage_ms_mean']
print('%-10s %-16s ms/step %.4f  ' % ('$d'[-10:], d['config']['workload'], d['ms_per_step']) + ' '.join('%s=%.3f' % (k[3:], v) for k, v in s.items()))")
    done
  done
done
