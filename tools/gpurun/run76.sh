#!/bin/bash
for m in memop host; do
  GSYS_COMPLETION=$m timeout 300 python tools/probe_dma.py > gpurun_out/probe76_$m.jsonl 2>&1
  GSYS_COMPLETION=$m timeout 120 python tools/sweep.py --staging device --chunk-kib 256 --blocks 296 > gpurun_out/sweep76_$m.jsonl 2>&1
done
