summ='import json,sys; d=json.loads(sys.stdin.readlines()[-1]); print(d["config"]["workload"], "value", d["value"], "ms", d["ms_per_step"])'
for rep in 1 2; do
for se in 0 65536; do
for drv in 1 2; do
echo -n "small=$se driver=$drv: "; timeout 900 python bench.py --steps 32 --warmup 3 --no-cpu-baseline --e2e-roots 0 --profile-roots 0 --small-edges $se --driver $drv 2>&1 | python -c "$summ"
done; done; done
