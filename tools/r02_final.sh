#!/bin/bash
# Round-2 final evidence on one B200: GPU tests, smoke, bench lines, reference arm, ncu
mkdir -p gpurun_out
timeout 1800 python -m pytest tests -m gpu -q > gpurun_out/f_pytest.txt 2>&1; echo "pytest rc=$?" >> gpurun_out/f_pytest.txt
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/f_smoke.txt 2>&1; echo "smoke rc=$?" >> gpurun_out/f_smoke.txt
for c in s24 s20 grid s24d s27; do
  timeout 1500 python bench.py --config $c > gpurun_out/f_bench_$c.json 2> gpurun_out/f_bench_$c.err; echo "$c rc=$?" >> gpurun_out/f_rc.txt
done
timeout 900 python bench.py --impl reference --steps 4 --warmup 3 > gpurun_out/f_bench_ref.json 2> gpurun_out/f_bench_ref.err; echo "ref rc=$?" >> gpurun_out/f_rc.txt
tools/profile.sh > gpurun_out/f_profile.log 2>&1; echo "profile rc=$?" >> gpurun_out/f_rc.txt
tail -2 gpurun_out/f_pytest.txt; cat gpurun_out/f_rc.txt
