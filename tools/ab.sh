#!/bin/bash
# A/B on one GPU box: tools/ab.sh DIR1,DIR2[,...] WORKLOAD...  (each a repo copy with a built .so,
# e.g. from tools/mkvariant.sh); two rounds of every variant per workload, interleaved
DIRS=$(echo $1 | tr ',' ' '); shift
for w in "$@"; do
  for rep in 1 2; do
    for d in $DIRS; do
      (cd $d && python bench.py --workload $w --no-cpu-baseline --no-e2e --no-closed-loop 2>/dev/null | tail -1 | python -c "
import json,sys; d=json.loads(sys.stdin.read()); s=d['stage_ms_mean']
print('%-10s %-16s ms/step %.4f  ' % ('$d'[-10:], d['config']['workload'], d['ms_per_step']) + ' '.join('%s=%.3f' % (k[3:], v) for k, v in s.items()))")
    done
  done
done
