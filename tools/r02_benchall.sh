#!/bin/bash
# Round-2 evidence: GPU tests, smoke, bench lines for the given configs -> gpurun_out/
#   tools/r02_benchall.sh [tests|notests] configs...
mkdir -p gpurun_out
T=$1; shift
if [ "$T" = tests ]; then
  timeout 1800 python -m pytest tests -m gpu -q > gpurun_out/b_pytest.txt 2>&1; echo "pytest rc=$?" >> gpurun_out/b_pytest.txt
  timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/b_smoke.txt 2>&1; echo "smoke rc=$?" >> gpurun_out/b_smoke.txt
fi
for c in "$@"; do
  timeout 1200 python bench.py --config $c > gpurun_out/b_bench_$c.json 2> gpurun_out/b_bench_$c.err
  echo "$c rc=$?" >> gpurun_out/b_rc.txt
done
tail -2 gpurun_out/b_pytest.txt 2>/dev/null; cat gpurun_out/b_rc.txt
