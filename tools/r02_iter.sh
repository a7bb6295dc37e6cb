#!/bin/bash
# one iteration: parity subset, A/B vs ablib/base.so on the given configs, per-level times
#   tools/r02_iter.sh "<pytest -k expr or ALL or NONE>" cfg...
mkdir -p gpurun_out
K=$1; shift
if [ "$K" = ALL ]; then timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/i_pytest.txt 2>&1
elif [ "$K" != NONE ]; then timeout 1500 python -m pytest tests -m gpu -x -q -k "$K" > gpurun_out/i_pytest.txt 2>&1; fi
tail -3 gpurun_out/i_pytest.txt 2>/dev/null
for c in "$@"; do
  tools/r02_ab.sh $c 32 ablib/base.so > /dev/null 2>&1
  timeout 300 python tools/level_times.py --config $c --roots 4 > gpurun_out/i_lt_$c.txt 2>&1
done
cat gpurun_out/ab_*.txt
