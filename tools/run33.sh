#!/bin/bash
for tool in memcheck racecheck synccheck; do
  timeout 900 compute-sanitizer --tool $tool --print-limit 20 python tools/sanitize_small.py > gpurun_out/san_$tool.log 2>&1; echo rc=$? >> gpurun_out/san_$tool.log
done
