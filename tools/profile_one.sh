#!/bin/bash
# ncu --set full on one kernel of the s24 bench: tools/profile_one.sh <name> <regex> [skip] [count]
name=$1; rx=$2; skip=${3:-0}; cnt=${4:-2}
mkdir -p gpurun_out
timeout 900 ncu --set full --clock-control none --import-source on --kernel-name-base demangled \
    -k "regex:$rx" -s $skip -c $cnt -o gpurun_out/prof_$name -f \
    python bench.py --steps 2 --warmup 3 --no-cpu-baseline --e2e-roots 0 --profile-roots 0 --driver 1 \
    > gpurun_out/prof_$name.txt 2>&1
