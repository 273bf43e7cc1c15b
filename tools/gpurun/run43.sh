#!/bin/bash
timeout 300 python tools/scan_bench.py 512 256 20 >> gpurun_out/scan43.jsonl 2>> gpurun_out/scan43.err
timeout 600 python -m pytest tests -q -m gpu -x -k "scan or wordcount" > gpurun_out/pytest43.log 2>&1; echo rc=$? >> gpurun_out/pytest43.log
timeout 600 ncu --set full --clock-control none --import-source on -k regex:scan_kernel -s 1 -c 1 -o gpurun_out/prof_scan43 python tools/scan_bench.py 512 256 2 > gpurun_out/ncu_scan43.log 2>&1; echo rc=$? >> gpurun_out/ncu_scan43.log
