#!/bin/bash
GSYS_SCAN_LD=3 timeout 300 python tools/zc_probe2.py > gpurun_out/zc21.jsonl 2> gpurun_out/zc21.err
out=gpurun_out/sweep21.jsonl; : > $out
python -c "import inputs; inputs.make_corpus(512, 16<<20)" 2>&1 | tail -1
for ld in 0 3 1; do
  GSYS_WC_LD=$ld timeout 120 python tools/sweep.py --staging host --chunk-kib 256 --blocks 296 >> $out 2>>gpurun_out/sweep21.err
done
GSYS_WC_LD=0 timeout 120 python tools/sweep.py --staging host --chunk-kib 256 --blocks 148 >> $out 2>>gpurun_out/sweep21.err
GSYS_WC_LD=0 timeout 120 python tools/sweep.py --staging host --chunk-kib 512 --blocks 296 >> $out 2>>gpurun_out/sweep21.err
