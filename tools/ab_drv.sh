#!/bin/bash
# A/B: previous build vs current build x {host loop, graph} (s24) + grid
summ='import json,sys; d=json.loads(sys.stdin.readlines()[-1]); print(d["config"]["workload"], "value", d["value"], "ms", d["ms_per_step"], json.dumps({k:v["avg_ms"] for k,v in d["kernels"].items()}))'
run() { echo -n "$1: "; env $1 timeout 900 python bench.py --steps 32 --warmup 3 --no-cpu-baseline --e2e-roots 0 --profile-roots ${PROF:-4} $2 2>&1 | python -c "$summ"; }
run "XBFS_LIB=ablib/libxbfs_prev.so"
run "X=1" "--driver 1"
run "X=2" "--driver 2"
run "XBFS_LIB=ablib/libxbfs_prev.so"
run "X=1" "--driver 1"
run "X=2" "--driver 2"
PROF=0 XBFS_ALLOW_SHORT_WARMUP=1 run "X=1" "--driver 1 --config grid --steps 2 --warmup 1"
PROF=0 XBFS_ALLOW_SHORT_WARMUP=1 run "X=2" "--driver 2 --config grid --steps 2 --warmup 1"
