#!/bin/bash
# alpha sweep on the in-tree library (s24, 48 roots, 2 reps)
out=gpurun_out/alpha.txt; : > $out
for rep in 1 2; do for al in 0.04 0.02 0.01 0.06; do
  r=$(timeout 600 python bench.py --config s24 --steps 48 --warmup 3 --alpha $al --no-cpu-baseline --e2e-roots 0 --profile-roots 0 --no-validate 2>&1 | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(d['value'], d['ms_per_step'])")
  echo "$rep alpha=$al $r" >> $out
done; done
cat $out
