#!/bin/bash
timeout 900 python -m pytest tests -m gpu -q -x > gpurun_out/pytest16.log 2>&1; echo rc=$? >> gpurun_out/pytest16.log
timeout 300 python tools/zc_probe.py > gpurun_out/zc16.jsonl 2> gpurun_out/zc16.err
timeout 600 python bench.py > gpurun_out/bench16.json 2> gpurun_out/bench16.err
timeout 900 ncu --set full --clock-control none --import-source on -k regex:scan_kernel -s 1 -c 1 -o gpurun_out/prof_scan16 python tools/prof_scan.py > gpurun_out/ncu_scan16.log 2>&1; echo rc=$? >> gpurun_out/ncu_scan16.log
