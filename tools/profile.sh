#!/bin/bash
# ncu evidence for the bench command (run under gpurun; 1 GPU).  Writes gpurun_out/.
set -x
mkdir -p gpurun_out
CMD="python bench.py --steps 2 --warmup 3 --no-cpu-baseline --e2e-roots 0 --profile-roots 0 --driver 1 $*"
# every launch with its device time (cold-cache, serialised: compare SHARES)
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv \
    --log-file gpurun_out/launches.csv $CMD > gpurun_out/launches_stdout.txt 2>&1
# full sections for the top kernels (skip warm-up launches)
timeout 900 ncu --set full --clock-control none --import-source on -k regex:bu_traverse -s 3 -c 2 \
    -o gpurun_out/prof_bu -f $CMD > gpurun_out/prof_bu.txt 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:td_expand -s 6 -c 3 \
    -o gpurun_out/prof_td -f $CMD > gpurun_out/prof_td.txt 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_generate -s 2 -c 2 \
    -o gpurun_out/prof_gen -f $CMD > gpurun_out/prof_gen.txt 2>&1
