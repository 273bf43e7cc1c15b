#!/bin/bash
timeout 1500 python -m pytest tests -m gpu -q -x > gpurun_out/pytest41.log 2>&1; echo rc=$? >> gpurun_out/pytest41.log
for m in host memop; do
  GSYS_COMPLETION=$m timeout 300 python tools/probe_dma.py > gpurun_out/probe41_$m.jsonl 2>&1
  GSYS_COMPLETION=$m timeout 120 python tools/sweep.py --staging device --chunk-kib 256 --blocks 296 > gpurun_out/sweep41_$m.jsonl 2>&1
  GSYS_COMPLETION=$m timeout 120 python tools/sweep.py --staging device --chunk-kib 1024 --blocks 296 >> gpurun_out/sweep41_$m.jsonl 2>&1
done
timeout 900 python bench.py --mode syscalls > gpurun_out/sys41.json 2> gpurun_out/sys41.err
