#!/bin/bash
# A/B several libxbfs.so builds by per-BFS device time (persistent driver level stamps):
#   tools/ab_levels.sh "<lib> <lib> ..." [roots] [extra level_times opts]
LIBS=$1; R=${2:-8}; shift; shift
for rep in 1 2; do
  for L in $LIBS; do
    echo -n "$L: "
    XBFS_LIB=$L python tools/level_times.py --roots $R $* | grep "^root" | python -c "
import sys,re
t=[];l=[]
for line in sys.stdin:
    m=re.search(r'([0-9.]+) us total, levels sum ([0-9.]+)',line); t.append(float(m.group(1))); l.append(float(m.group(2)))
print('mean total %.1f levels %.1f other %.1f' % (sum(t)/len(t), sum(l)/len(l), (sum(t)-sum(l))/len(t)))"
  done
done
