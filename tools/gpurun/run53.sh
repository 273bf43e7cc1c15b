#!/bin/bash
for p in 4096 1024 256 64; do GSYS_POLL_NS_HOST=$p timeout 120 python tools/lat_probe.py >> gpurun_out/lat53.jsonl 2>> gpurun_out/lat53.err; done
