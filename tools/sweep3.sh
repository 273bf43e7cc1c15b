#!/bin/bash
out=gpurun_out/sweep3.jsonl
: > $out
python -c "import inputs; inputs.make_corpus(512, 16<<20)" 2>&1 | tail -1
for st in device host; do
  for c in 256 1024; do
   GSYS_THREADS=12 timeout 120 python tools/sweep.py --staging $st --chunk-kib $c --cmax 8 >> $out 2>>gpurun_out/sweep3.err
  done
done
timeout 600 python bench.py --staging host > gpurun_out/bench3.json 2> gpurun_out/bench3.err
cat $out
