#!/bin/bash
out=gpurun_out/sweep10.jsonl; : > $out
python -c "import inputs; inputs.make_corpus(512, 16<<20)" 2>&1 | tail -1
for t in 12 15; do for b in 148 296 592; do for c in 128 256; do
  GSYS_THREADS=$t timeout 120 python tools/sweep.py --staging host --chunk-kib $c --blocks $b >> $out 2>>gpurun_out/sweep10.err
done; done; done
