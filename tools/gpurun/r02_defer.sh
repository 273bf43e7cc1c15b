#!/bin/bash
# WI non-blocking device-buffer preads vs the per-worker deferred store size (GSYS_DEFER_MB)
cd "$GRAFT_REPO_ROOT" || exit 1
O=gpurun_out
for mb in 16 48 96; do
  GSYS_DEFER_MB=$mb timeout 300 python tools/nb_probe.py | sed "s/^{/{\"defer_mb\": $mb, /" >> $O/r02_defer.jsonl
done
cat $O/r02_defer.jsonl
