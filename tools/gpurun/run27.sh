#!/bin/bash
# mixed staging sweep: SM zero-copy + copy-engine DMA on the host link
python -c "import inputs; inputs.make_corpus(512, 16<<20)" 2>&1 | tail -1
for c in 256 1024; do
  for st in host device; do
    timeout 120 python tools/sweep.py --staging $st --chunk-kib $c --blocks 296 >> gpurun_out/sweep27.jsonl 2>>gpurun_out/sweep27.err
  done
  for d in 1 2 3 4 6 8; do
    timeout 120 python tools/sweep.py --staging mixed --dev16 $d --chunk-kib $c --blocks 296 >> gpurun_out/sweep27.jsonl 2>>gpurun_out/sweep27.err
  done
done
for b in 148 444 592; do
  timeout 120 python tools/sweep.py --staging mixed --dev16 3 --chunk-kib 256 --blocks $b >> gpurun_out/sweep27.jsonl 2>>gpurun_out/sweep27.err
done
