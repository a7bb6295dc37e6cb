#!/bin/bash
# A/B two builds of libxbfs.so on the same box: tools/ab_lib.sh <libA> <libB> [bench args]
A=$1; B=$2; shift 2
summ='import json,sys; d=json.loads(sys.stdin.readlines()[-1]); print(d["config"]["workload"], "value", d["value"], "ms", d["ms_per_step"])'
for rep in 1 2; do
  for L in $A $B; do
    echo -n "$L: "; XBFS_LIB=$L timeout 900 python bench.py --steps 32 --warmup 3 --no-cpu-baseline --e2e-roots 0 --profile-roots 0 $* 2>&1 | python -c "$summ"
  done
done
