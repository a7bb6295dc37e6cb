summ='import json,sys; d=json.loads(sys.stdin.readlines()[-1]); print(d["config"]["workload"], "value", d["value"], "ms", d["ms_per_step"])'
for L in $*; do
  echo -n "$L: "; XBFS_LIB=$L timeout 600 python bench.py --config grid --steps 4 --warmup 3 --no-cpu-baseline --e2e-roots 0 --profile-roots 0 2>&1 | python -c "$summ"
done
