#!/bin/bash
# config 1 vs the completion-poll knobs: learned pre-poll sleep on/off, host poll interval
cd "$GRAFT_REPO_ROOT" || exit 1
O=gpurun_out
for hint in 1 0; do for pns in 256 64; do
  GSYS_SLEEP_HINT=$hint GSYS_POLL_NS_HOST=$pns C1_CHUNKS=64,128 timeout 300 python tools/config1_sweep.py 2>/dev/null | \
    python -c "import sys,json
for l in sys.stdin:
    d=json.loads(l); d['sleep_hint']=$hint; d['poll_ns_host']=$pns; print(json.dumps(d))" >> $O/r02_c1poll.jsonl
done; done
cut -c1-220 $O/r02_c1poll.jsonl
