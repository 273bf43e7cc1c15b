#!/bin/bash
# config 1 vs service knobs: split threshold (B14) and service thread count, host + device staging
cd "$GRAFT_REPO_ROOT" || exit 1
O=gpurun_out
for th in 14 8; do for sk in 128 32 16; do
  GSYS_THREADS=$th GSYS_SPLIT_KB=$sk C1_CHUNKS=128,64 timeout 300 python tools/config1_sweep.py 2>/dev/null | \
    python -c "import sys,json
for l in sys.stdin:
    d=json.loads(l); d['threads']=$th; d['split_kb']=$sk; print(json.dumps(d))" >> $O/r02_c1env.jsonl
done; done
cat $O/r02_c1env.jsonl
