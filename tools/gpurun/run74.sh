#!/bin/bash
timeout 300 python tools/probe_dma.py > gpurun_out/probe74.jsonl 2>&1
timeout 900 python bench.py --mode syscalls --cell-ms 60 > gpurun_out/sys74.json 2> gpurun_out/sys74.err
timeout 120 python tools/sweep.py --staging device --chunk-kib 256 --blocks 296 > gpurun_out/sweep74.jsonl 2>&1
