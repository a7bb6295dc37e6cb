#!/bin/bash
# quick GPU check: parity tests + s24 bench summary + grid per-level cost
timeout 900 python -m pytest tests -x -q -m gpu 2>&1 | tail -3
summ='import json,sys; d=json.loads(sys.stdin.readlines()[-1]); print(d["config"]["workload"], "value", d["value"], "ms", d["ms_per_step"], "model_frac", d["roofline_model"]["frac"], d["strategies"][:2]); print(json.dumps({k:(v["avg_ms"],v["gbs"]) for k,v in d["kernels"].items()}))'
timeout 900 python bench.py --steps 32 --warmup 3 --no-cpu-baseline $* 2>&1 | python -c "$summ"
XBFS_ALLOW_SHORT_WARMUP=1 timeout 600 python bench.py --config grid --steps 2 --warmup 1 --no-cpu-baseline --e2e-roots 0 --profile-roots 0 $* 2>&1 | python -c "$summ"
