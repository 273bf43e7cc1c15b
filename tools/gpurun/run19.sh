#!/bin/bash
out=gpurun_out/sweep19.jsonl; : > $out
python -c "import inputs; inputs.make_corpus(512, 16<<20)" 2>&1 | tail -1
for b in 148 296; do
  timeout 120 python tools/sweep.py --staging host --chunk-kib 256 --blocks $b >> $out 2>>gpurun_out/sweep19.err
done
GSYS_WC_LD=0 timeout 120 python tools/sweep.py --staging host --chunk-kib 256 --blocks 296 >> $out 2>>gpurun_out/sweep19.err
timeout 120 python tools/sweep.py --staging host --chunk-kib 256 --blocks 296 --threads 128 >> $out 2>>gpurun_out/sweep19.err
timeout 120 python tools/sweep.py --staging device --chunk-kib 1024 --blocks 296 >> $out 2>>gpurun_out/sweep19.err
