#!/bin/bash
for th in 512 384; do timeout 300 python tools/scan_bench.py $th 256 20 >> gpurun_out/scan42.jsonl 2>> gpurun_out/scan42.err; done
timeout 600 python -m pytest tests -q -m gpu -x > gpurun_out/pytest42.log 2>&1; echo rc=$? >> gpurun_out/pytest42.log
timeout 600 ncu --set full --clock-control none --import-source on -k regex:scan_kernel -s 1 -c 1 -o gpurun_out/prof_scan42 python tools/scan_bench.py 512 256 2 > gpurun_out/ncu_scan42.log 2>&1; echo rc=$? >> gpurun_out/ncu_scan42.log
