#!/bin/bash
# host-staging sweep: chunk x work-groups x service threads (profile counters on)
python -c "import inputs; inputs.make_corpus(512, 16<<20)" > /dev/null 2>&1
for cfg in "256 296 14" "128 296 14" "64 592 14" "128 592 14" "512 296 14" "256 148 14" "256 444 14" "256 296 15" "256 296 12" "256 296 10"; do
  set -- $cfg
  GSYS_THREADS=$3 timeout 300 python tools/sweep.py --staging host --chunk-kib $1 --blocks $2 --steps 3 >> gpurun_out/sweep47.jsonl 2>> gpurun_out/sweep47.err
done
