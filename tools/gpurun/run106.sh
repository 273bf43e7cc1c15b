#!/bin/bash
for k in getrusage pread; do
  timeout 900 ncu --set full --import-source on --clock-control none --replay-mode application -k regex:bench_kernel -c 1 -o gpurun_out/prof_calls_$k python tools/prof_calls.py $k > gpurun_out/ncu_calls_$k.log 2>&1; echo rc=$? >> gpurun_out/ncu_calls_$k.log
done
