#!/bin/bash
timeout 1200 python -m pytest tests/test_gpu.py -m gpu -q -x -k "nonblocking or wordcount_config1 or injected" > gpurun_out/pytest79.log 2>&1; echo rc=$? >> gpurun_out/pytest79.log
for i in 1 2; do
  for nb in 0 1; do
    timeout 120 python tools/sweep.py --staging host --chunk-kib 256 --blocks 296 --steps 5 --nonblocking $nb >> gpurun_out/sweep79.jsonl 2>&1
  done
done
for c in 128 512; do timeout 120 python tools/sweep.py --staging host --chunk-kib $c --blocks 296 --steps 5 --nonblocking 1 >> gpurun_out/sweep79.jsonl 2>&1; done
for b in 148 444; do timeout 120 python tools/sweep.py --staging host --chunk-kib 256 --blocks $b --steps 5 --nonblocking 1 >> gpurun_out/sweep79.jsonl 2>&1; done
timeout 120 python tools/sweep.py --staging device --chunk-kib 256 --blocks 296 --steps 5 --nonblocking 1 >> gpurun_out/sweep79.jsonl 2>&1
