#!/bin/bash
for th in 512 256 384; do timeout 300 python tools/scan_bench.py $th 256 20 >> gpurun_out/scan41.jsonl 2>> gpurun_out/scan41.err; done
timeout 300 python tools/scan_bench.py 512 64 20 >> gpurun_out/scan41.jsonl 2>> gpurun_out/scan41.err
timeout 600 python -m pytest tests -q -m gpu -x > gpurun_out/pytest41.log 2>&1; echo rc=$? >> gpurun_out/pytest41.log
timeout 600 ncu --set full --clock-control none --import-source on -k regex:scan_kernel -s 1 -c 1 -o gpurun_out/prof_scan41 python tools/scan_bench.py 512 256 2 > gpurun_out/ncu_scan41.log 2>&1; echo rc=$? >> gpurun_out/ncu_scan41.log
