#!/bin/bash
timeout 900 python -m pytest tests -m gpu -q -x -k "injected or pull or matrix" > gpurun_out/pytest60.log 2>&1; echo rc=$? >> gpurun_out/pytest60.log
timeout 900 ncu --set full --clock-control none --import-source on -k regex:scan_kernel -s 1 -c 1 -o gpurun_out/prof_scan60 python tools/prof_scan.py > gpurun_out/ncu_scan60.log 2>&1; echo rc=$? >> gpurun_out/ncu_scan60.log
for t in 12 16; do
  GSYS_THREADS=$t timeout 900 python bench.py --mode syscalls --cell-ms 60 > gpurun_out/sys60_t$t.json 2> gpurun_out/sys60_t$t.err
done
