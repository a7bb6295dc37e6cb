#!/bin/bash
# compute-sanitizer over tools/sanitize.py on the current build (drivers 1 + persistent, directed, dist 1 rank)
mkdir -p gpurun_out
export SANITIZE_DRIVERS=1 SANITIZE_PERSIST=1 SANITIZE_DIST=1
for t in memcheck initcheck racecheck synccheck; do
  timeout 1200 compute-sanitizer --tool $t --error-exitcode 9 python tools/sanitize.py > gpurun_out/san_$t.txt 2>&1
  echo "$t rc=$? $(grep -E 'ERROR SUMMARY|RACECHECK SUMMARY' gpurun_out/san_$t.txt | tail -1)" >> gpurun_out/san_rc.txt
done
cat gpurun_out/san_rc.txt
