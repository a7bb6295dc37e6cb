summ='import json,sys; d=json.loads(sys.stdin.readlines()[-1]); print("value", d["value"], "ms", d["ms_per_step"])'
for rep in 1 2; do for drv in 1 2; do echo -n "driver=$drv: "; timeout 900 python bench.py --steps 32 --warmup 3 --no-cpu-baseline --e2e-roots 0 --profile-roots 0 --driver $drv 2>&1 | python -c "$summ"; done; done
