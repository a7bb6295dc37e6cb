#!/bin/bash
# one k_persist --set full capture (source-level) on the s24 bench command
mkdir -p gpurun_out
CFG=${1:-s24}
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_persist -s 3 -c 1 \
    -o gpurun_out/p_persist -f python bench.py --config $CFG --steps 1 --warmup 3 --no-cpu-baseline --e2e-roots 0 --profile-roots 0 > gpurun_out/p_ncu.txt 2>&1
tail -2 gpurun_out/p_ncu.txt
