#!/bin/bash
# one source-level ncu capture of k_persist for the s24 bench command, launch index $1 (3 = first timed root)
mkdir -p gpurun_out
S=${1:-3}; CFG=${2:-s24}; TAG=${3:-p}
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_persist -s $S -c 1 \
    -o gpurun_out/${TAG}_persist_$CFG -f python bench.py --config $CFG --steps 2 --warmup 3 --no-cpu-baseline --e2e-roots 0 --profile-roots 0 --no-validate > gpurun_out/${TAG}_ncu_$CFG.txt 2>&1
tail -1 gpurun_out/${TAG}_ncu_$CFG.txt | cut -c1-300
