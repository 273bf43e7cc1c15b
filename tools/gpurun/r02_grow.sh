#!/bin/bash
# deferred-pull overflow store (GSYS_DEFER_GROW_MB): tests, then WI/WG non-blocking rates with and without it
cd "$GRAFT_REPO_ROOT" || exit 1
O=gpurun_out
timeout 900 python -m pytest tests -m gpu -x -q -k "deferred or nonblocking or token or pull" > $O/r02g_tests.log 2>&1; tail -2 $O/r02g_tests.log
for g in 0 64; do
  GSYS_DEFER_GROW_MB=$g timeout 300 python tools/nb_probe.py | sed "s/^{/{\"grow_mb\": $g, /" >> $O/r02_defer_grow.jsonl
done
cat $O/r02_defer_grow.jsonl | cut -c1-200
