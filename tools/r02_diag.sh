#!/bin/bash
# per-level device times + one source-level ncu capture of k_persist per config
mkdir -p gpurun_out
for c in "$@"; do
  timeout 600 python tools/level_times.py --config $c --roots 6 > gpurun_out/d_lt_$c.txt 2>&1
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_persist -s 4 -c 1 \
    -o gpurun_out/d_persist_$c -f python bench.py --config $c --steps 2 --warmup 3 --no-cpu-baseline --e2e-roots 0 --profile-roots 0 --no-validate > gpurun_out/d_ncu_$c.txt 2>&1
  echo "$c done" >> gpurun_out/d_rc.txt
done
