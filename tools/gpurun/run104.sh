#!/bin/bash
for p in 64 128 256 512; do
  GSYS_POLL_NS_HOST=$p timeout 600 python tools/phase_probe.py > gpurun_out/poll104_$p.jsonl 2>&1
done
