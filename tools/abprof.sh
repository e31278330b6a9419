#!/bin/bash
# tools/abprof.sh WORKLOAD KERNEL_REGEX SKIP COUNT DIR... : a few ncu metrics of the same launches per checkout
W=$1; K=$2; S=$3; C=$4; shift 4
M=dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum,lts__t_sector_hit_rate.pct,lts__t_sectors_srcunit_tex_op_read.sum,lts__t_sectors_srcunit_tex_op_atom.sum,lts__t_sectors_srcunit_tex_op_red.sum,lts__t_sectors_srcunit_tex_op_write.sum,sm__warps_active.avg.pct_of_peak_sustained_active
for d in "$@"; do
  echo "== $d $W"
  (cd $d; LTPG_NO_CLOCKS=1 /usr/local/cuda/bin/ncu --csv --metrics $M -k "regex:$K" -s $S -c $C python bench.py --workload $W --steps 2 --warmup 3 --no-cpu-baseline --no-e2e 2>/dev/null | python -c "
import csv,sys
rows=[r for r in csv.reader(l for l in sys.stdin if l.startswith('\"'))]
h=rows[0]; ki=h.index('Kernel Name'); mi=h.index('Metric Name'); vi=h.index('Metric Value'); ui=h.index('Metric Unit'); ii=h.index('ID')
cur=None
for r in rows[1:]:
  if r[ii]!=cur: cur=r[ii]; print('  #%s %s' % (cur, r[ki][:60]))
  print('     %-55s %14s %s' % (r[mi], r[vi], r[ui]))
")
done
