summ='import json,sys; d=json.loads(sys.stdin.readlines()[-1]); print("value", d["value"], "ms", d["ms_per_step"], json.dumps({k:v["avg_ms"] for k,v in d["kernels"].items()}))'
run() { echo -n "$1: "; env $1 timeout 900 python bench.py --steps 32 --warmup 3 --no-cpu-baseline --e2e-roots 0 --profile-roots 4 2>&1 | python -c "$summ"; }
run "XBFS_LIB=ablib/libxbfs_prev.so"
run "X=0"
run "XBFS_GRID_BU=8"
run "XBFS_GRID_GEN=8"
run "XBFS_GRID_EXPAND=4"
run "XBFS_GRID_BU=8 XBFS_GRID_GEN=8 XBFS_GRID_EXPAND=4"
run "XBFS_LIB=ablib/libxbfs_prev.so"
