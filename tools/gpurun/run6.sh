#!/bin/bash
out=gpurun_out/sweep6.jsonl; : > $out
python -c "import inputs; inputs.make_corpus(512, 16<<20)" 2>&1 | tail -1
for st in host device; do for c in 256 1024; do
  GSYS_THREADS=12 timeout 120 python tools/sweep.py --staging $st --chunk-kib $c >> $out 2>>gpurun_out/sweep6.err
done; done
GSYS_THREADS=12 timeout 120 python tools/sweep.py --staging host --chunk-kib 256 --blocks 1184 >> $out 2>>gpurun_out/sweep6.err
