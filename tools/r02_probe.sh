#!/bin/bash
# round-2 baseline probe: per-level times (s24, s20) + k_persist source-level stall capture
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > gpurun_out/p_smi.txt
timeout 600 python tools/level_times.py --config s24 --roots 4 > gpurun_out/p_lt_s24.txt 2>&1
timeout 600 python tools/level_times.py --config s20 --roots 2 > gpurun_out/p_lt_s20.txt 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_persist -s 3 -c 1 \
    -o gpurun_out/p_persist -f python bench.py --steps 1 --warmup 3 --no-cpu-baseline --e2e-roots 0 --profile-roots 0 > gpurun_out/p_ncu.txt 2>&1
echo done
