#!/bin/bash
# A/B several builds on one box: tools/ab_multi.sh "lib1 lib2 ..." [bench args]
LIBS=$1; shift
summ='import json,sys; d=json.loads(sys.stdin.readlines()[-1]); print("value", d["value"], "ms", d["ms_per_step"], json.dumps({k:v["avg_ms"] for k,v in d.get("kernels",{}).items() if k in ("bu_traverse","td_expand_ss","td_expand_sf","generate_post")}))'
for rep in 1 2; do
  for L in $LIBS; do
    echo -n "$L: "; XBFS_LIB=$L timeout 900 python bench.py --steps 32 --warmup 3 --no-cpu-baseline --e2e-roots 0 --profile-roots 2 "$@" 2>&1 | python -c "$summ"
  done
done
