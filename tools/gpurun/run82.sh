#!/bin/bash
for i in 1 2 3; do timeout 120 python tools/scan_bench.py 512 256 30; done > gpurun_out/scan82.jsonl 2>&1
timeout 900 python -m pytest tests -m gpu -q -x -k "scan or wordcount" > gpurun_out/pytest82.log 2>&1; echo rc=$? >> gpurun_out/pytest82.log
