#!/bin/bash
# ncu evidence for the bench command (run under gpurun; 1 GPU).  Writes gpurun_out/.
#   tools/profile.sh [extra bench args]
set -x
mkdir -p gpurun_out
CMD="python bench.py --steps 2 --warmup 3 --no-cpu-baseline --e2e-roots 0 --profile-roots 0 $*"
# every launch with its device time (cold-cache, serialised: compare SHARES)
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv \
    --log-file gpurun_out/launches.csv $CMD > gpurun_out/launches_stdout.txt 2>&1
# full sections for the timed persistent-kernel launches (skip the 3 warm-up BFS)
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_persist -s 3 -c 2 \
    -o gpurun_out/prof_persist -f $CMD > gpurun_out/prof_persist.txt 2>&1
