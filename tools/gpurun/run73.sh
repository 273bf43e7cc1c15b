#!/bin/bash
timeout 1500 python -m pytest tests -m gpu -q -x > gpurun_out/pytest73.log 2>&1; echo rc=$? >> gpurun_out/pytest73.log
timeout 300 python tools/probe_dma.py > gpurun_out/probe73.jsonl 2>&1
timeout 900 python bench.py --mode syscalls > gpurun_out/sys73.json 2> gpurun_out/sys73.err
timeout 120 python tools/sweep.py --staging device --chunk-kib 256 --blocks 296 > gpurun_out/sweep73.jsonl 2>&1
