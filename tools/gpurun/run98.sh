#!/bin/bash
python -c "import inputs; inputs.make_corpus(512, 16<<20)" > /dev/null 2>&1
for c in 256 1024; do for b in 148 296 592; do
  timeout 120 python tools/sweep.py --staging device --chunk-kib $c --blocks $b --steps 3 >> gpurun_out/dev98.jsonl 2>&1
done; done
GSYS_THREADS=16 timeout 120 python tools/sweep.py --staging device --chunk-kib 256 --blocks 296 --steps 3 >> gpurun_out/dev98.jsonl 2>&1
GSYS_BOUNCE_MB=128 timeout 120 python tools/sweep.py --staging device --chunk-kib 256 --blocks 296 --steps 3 >> gpurun_out/dev98.jsonl 2>&1
