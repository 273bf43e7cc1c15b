#!/bin/bash
timeout 900 python -m pytest tests -m gpu -q -x > gpurun_out/pytest_gpu.log 2>&1; echo rc=$? >> gpurun_out/pytest_gpu.log
GSYS_THREADS=12 timeout 300 python tools/probe_calls.py getrusage > gpurun_out/probe4.jsonl 2> gpurun_out/probe4.err
out=gpurun_out/sweep4.jsonl; : > $out
for st in host device; do for c in 256 1024; do
  GSYS_THREADS=12 timeout 120 python tools/sweep.py --staging $st --chunk-kib $c >> $out 2>>gpurun_out/sweep4.err
done; done
GSYS_THREADS=14 timeout 120 python tools/sweep.py --staging host --chunk-kib 256 >> $out 2>>gpurun_out/sweep4.err
GSYS_THREADS=14 GSYS_POLL_NS_MAX=8192 timeout 120 python tools/sweep.py --staging host --chunk-kib 256 >> $out 2>>gpurun_out/sweep4.err
