#!/bin/bash
timeout 900 python -m pytest tests -m gpu -q -x -k "scan" > gpurun_out/pytest88.log 2>&1; echo rc=$? >> gpurun_out/pytest88.log
timeout 900 ncu --set full --clock-control none --import-source on -k regex:scan_kernel -s 1 -c 1 -o gpurun_out/prof_scan88 python tools/prof_scan.py > gpurun_out/ncu_scan88.log 2>&1; echo rc=$? >> gpurun_out/ncu_scan88.log
timeout 900 python bench.py > gpurun_out/bench88.json 2> gpurun_out/bench88.err; echo rc=$? >> gpurun_out/bench88.err
