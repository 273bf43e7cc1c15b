#!/bin/bash
# is the per-caller latency growth host-memory polling contention?  hint off, long poll intervals
for p in 256 8000 20000 50000; do
  GSYS_SLEEP_HINT=0 GSYS_POLL_NS_HOST=$p timeout 300 python tools/probe_calls.py getrusage > gpurun_out/probe38_$p.jsonl 2>&1
done
