#!/bin/bash
# after the warp-cooperative token scan: full GPU suite, memcheck + racecheck of the small run
cd "$GRAFT_REPO_ROOT" || exit 1
O=gpurun_out
timeout 1200 python -m pytest tests -m gpu -x -q > $O/r02v_gputest.log 2>&1; tail -2 $O/r02v_gputest.log
for tool in memcheck racecheck; do
  timeout 1500 compute-sanitizer --tool $tool --print-limit 20 python tools/sanitize_small.py > $O/r02v_sanitize_$tool.log 2>&1
  echo "$tool rc=$?"; grep -E "ERROR SUMMARY|RACECHECK SUMMARY|hazard" $O/r02v_sanitize_$tool.log | tail -3
done
