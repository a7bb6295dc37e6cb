#!/bin/bash
# GPU check: parity tests (optionally a -k filter), smoke, per-level times
mkdir -p gpurun_out
K=${1:-}
if [ -n "$K" ]; then
  timeout 1500 python -m pytest tests -m gpu -x -q -k "$K" > gpurun_out/c_pytest.txt 2>&1
else
  timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/c_pytest.txt 2>&1
fi
echo "pytest rc=$?" >> gpurun_out/c_pytest.txt
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/c_smoke.txt 2>&1
timeout 600 python tools/level_times.py --config s24 --roots 4 > gpurun_out/c_lt_s24.txt 2>&1
tail -3 gpurun_out/c_pytest.txt
