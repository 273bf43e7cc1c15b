#!/bin/bash
# doorbell fence variants: acq_rel (default), sc (round-1 original), none (diagnostic)
for v in default sc nofence; do
  if [ $v = default ]; then L=""; else L=$PWD/tools/variants/libgsys_$v.so; fi
  GSYS_LIB=$L timeout 300 python tools/probe_calls.py getrusage pread > gpurun_out/probe37_$v.jsonl 2>&1
done
