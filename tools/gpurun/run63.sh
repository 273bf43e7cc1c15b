#!/bin/bash
# compute-sanitizer over every kernel incl. the pull path
for t in memcheck racecheck synccheck; do
  timeout 900 compute-sanitizer --tool $t --target-processes all python tools/sanitize_small.py > gpurun_out/san63_$t.log 2>&1; echo "rc=$?" >> gpurun_out/san63_$t.log
done
