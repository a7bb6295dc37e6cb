#!/bin/bash
# A/B several builds of libxbfs.so on one box: tools/ab_many.sh "<lib> <lib> ..." [bench args]
LIBS=$1; shift
summ='import json,sys; d=json.loads(sys.stdin.readlines()[-1]); r=d["roofline"] or {}; print("value", d["value"], "ms", d["ms_per_step"], "phases", json.dumps(r.get("phases")))'
for rep in 1 2; do
  for L in $LIBS; do
    echo -n "$L: "; XBFS_LIB=$L timeout 900 python bench.py --steps 32 --warmup 3 --no-cpu-baseline --e2e-roots 0 --profile-roots 0 $* 2>&1 | python -c "$summ"
  done
done
