#!/bin/bash
# A/B on one box: bench (value, ms/BFS) for the in-tree library vs ablib/<name>.so, interleaved.
#   tools/r02_ab.sh [config] [steps] [libs...]
mkdir -p gpurun_out
CFG=${1:-s24}; STEPS=${2:-24}; shift 2; LIBS=${@:-ablib/libxbfs_r1.so}
out=gpurun_out/ab_$CFG.txt; : > $out
for rep in 1 2; do
  for lib in paper_conf_sc_yangls0w24_b200/libxbfs.so $LIBS; do
    r=$(XBFS_LIB=$lib timeout 600 python bench.py --config $CFG --steps $STEPS --warmup 3 --no-cpu-baseline \
        --e2e-roots 0 --profile-roots 0 --no-validate 2>&1 | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(d['value'], d['ms_per_step'], d['roofline']['frac'] if d.get('roofline') else None)" 2>&1)
    echo "$rep $lib $r" >> $out
  done
done
cat $out
