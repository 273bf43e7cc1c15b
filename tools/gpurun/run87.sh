#!/bin/bash
for i in 1 2; do
  for t in 512 704; do
    timeout 120 python tools/scan_bench.py $t 256 30 | sed "s/^{/{\"v\":\"x2\",/" >> gpurun_out/scan87.jsonl 2>&1
    GSYS_LIB=$PWD/tools/variants/libgsys_onechain.so timeout 120 python tools/scan_bench.py $t 256 30 | sed "s/^{/{\"v\":\"x1\",/" >> gpurun_out/scan87.jsonl 2>&1
  done
done
timeout 900 python -m pytest tests -m gpu -q -x -k "scan or wordcount" > gpurun_out/pytest87.log 2>&1; echo rc=$? >> gpurun_out/pytest87.log
for i in 1 2; do
  timeout 120 python tools/sweep.py --staging host --chunk-kib 256 --blocks 148 --steps 5 | sed "s/^{/{\"v\":\"x2\",/" >> gpurun_out/wc87.jsonl 2>&1
  GSYS_LIB=$PWD/tools/variants/libgsys_onechain.so timeout 120 python tools/sweep.py --staging host --chunk-kib 256 --blocks 148 --steps 5 | sed "s/^{/{\"v\":\"x1\",/" >> gpurun_out/wc87.jsonl 2>&1
done
