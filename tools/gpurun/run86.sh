#!/bin/bash
timeout 300 python tools/config1_probe.py > gpurun_out/c1_86.json 2>&1
timeout 1500 python -m pytest tests -m gpu -q -x > gpurun_out/pytest86.log 2>&1; echo rc=$? >> gpurun_out/pytest86.log
for i in 1 2; do timeout 120 python tools/sweep.py --staging host --chunk-kib 256 --blocks 148 --steps 5 >> gpurun_out/sweep86.jsonl 2>&1; done
timeout 900 python bench.py --mode syscalls --cell-ms 60 > gpurun_out/sys86.json 2> gpurun_out/sys86.err
