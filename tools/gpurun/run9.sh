#!/bin/bash
out=gpurun_out/sweep9.jsonl; : > $out
python -c "import inputs; inputs.make_corpus(512, 16<<20)" 2>&1 | tail -1
for ld in 1 3 0 2; do
  GSYS_WC_LD=$ld GSYS_THREADS=12 timeout 120 python tools/sweep.py --staging host --chunk-kib 256 >> $out 2>>gpurun_out/sweep9.err
done
for ld in 1 3; do
  GSYS_WC_LD=$ld GSYS_THREADS=12 timeout 120 python tools/sweep.py --staging device --chunk-kib 256 >> $out 2>>gpurun_out/sweep9.err
done
