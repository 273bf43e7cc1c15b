#!/bin/bash
out=gpurun_out/sweep2.jsonl
: > $out
python -c "import inputs; inputs.make_corpus(512, 16<<20)" 2>&1 | tail -1
for st in device host; do
 for c in 256 1024; do
  for cm in 8 64; do
   GSYS_THREADS=12 timeout 120 python tools/sweep.py --staging $st --chunk-kib $c --cmax $cm >> $out 2>>gpurun_out/sweep2.err
  done
 done
done
GSYS_THREADS=8 timeout 120 python tools/sweep.py --staging host --chunk-kib 256 --cmax 64 >> $out 2>>gpurun_out/sweep2.err
GSYS_THREADS=14 timeout 120 python tools/sweep.py --staging host --chunk-kib 256 --cmax 64 >> $out 2>>gpurun_out/sweep2.err
GSYS_THREADS=12 timeout 120 python tools/sweep.py --staging host --chunk-kib 64 --cmax 64 >> $out 2>>gpurun_out/sweep2.err
cat $out
