#!/bin/bash
timeout 900 python -m pytest tests -m gpu -q -x > gpurun_out/pytest18.log 2>&1; echo rc=$? >> gpurun_out/pytest18.log
timeout 300 python tools/zc_probe.py > gpurun_out/zc18.jsonl 2> gpurun_out/zc18.err
timeout 900 ncu --set full --clock-control none --import-source on -k regex:scan_kernel -s 1 -c 1 -o gpurun_out/prof_scan18 python tools/prof_scan.py > gpurun_out/ncu_scan18.log 2>&1; echo rc=$? >> gpurun_out/ncu_scan18.log
timeout 600 python bench.py --no-cpu-baseline > gpurun_out/bench18.json 2> gpurun_out/bench18.err
