#!/bin/bash
out=gpurun_out/sweep5.jsonl; : > $out
python -c "import inputs; inputs.make_corpus(512, 16<<20)" 2>&1 | tail -1
for ph in 2048 4096 16384; do
  GSYS_POLL_NS_HOST=$ph GSYS_THREADS=12 timeout 120 python tools/sweep.py --staging host --chunk-kib 256 >> $out 2>>gpurun_out/sweep5.err
done
GSYS_POLL_NS_HOST=8192 GSYS_THREADS=12 timeout 120 python tools/sweep.py --staging host --chunk-kib 1024 >> $out 2>>gpurun_out/sweep5.err
GSYS_POLL_NS_HOST=8192 GSYS_THREADS=12 timeout 120 python tools/sweep.py --staging host --chunk-kib 256 --blocks 148 >> $out 2>>gpurun_out/sweep5.err
GSYS_POLL_NS_HOST=4096 GSYS_THREADS=12 timeout 300 python tools/probe_calls.py getrusage > gpurun_out/probe5.jsonl 2> gpurun_out/probe5.err
