#!/bin/bash
timeout 900 python -m pytest tests -m gpu -q -x > gpurun_out/pytest23.log 2>&1; echo rc=$? >> gpurun_out/pytest23.log
GSYS_SCAN_LD=0 timeout 300 python tools/zc_probe2.py > gpurun_out/zc23.jsonl 2> gpurun_out/zc23.err
timeout 300 python tools/zc_probe.py >> gpurun_out/zc23.jsonl 2>> gpurun_out/zc23.err
out=gpurun_out/sweep23.jsonl; : > $out
for b in 148 296 592; do
  timeout 120 python tools/sweep.py --staging host --chunk-kib 256 --blocks $b >> $out 2>>gpurun_out/sweep23.err
done
timeout 120 python tools/sweep.py --staging device --chunk-kib 1024 --blocks 296 >> $out 2>>gpurun_out/sweep23.err
