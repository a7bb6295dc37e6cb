#!/bin/bash
# A/B of several library builds (in-tree + ablib/*.so given), interleaved, 2 reps:
#   tools/r02_abn.sh cfg steps lib...
mkdir -p gpurun_out
CFG=$1; STEPS=$2; shift 2
out=gpurun_out/abn_$CFG.txt; : > $out
for rep in 1 2; do
  for lib in paper_conf_sc_yangls0w24_b200/libxbfs.so "$@"; do
    r=$(XBFS_LIB=$lib timeout 600 python bench.py --config $CFG --steps $STEPS --warmup 3 --no-cpu-baseline \
        --e2e-roots 0 --profile-roots 0 --no-validate 2>&1 | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(d['value'], d['ms_per_step'], d['roofline']['frac'] if d.get('roofline') else None)" 2>&1)
    echo "$rep $(basename $lib) $r" >> $out
  done
done
cat $out
