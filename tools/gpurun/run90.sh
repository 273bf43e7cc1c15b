#!/bin/bash
for v in 0 1; do
  GSYS_SHARE_BURSTS=$v timeout 300 python tools/config1_probe.py > gpurun_out/c1_90_$v.json 2>&1
  GSYS_SHARE_BURSTS=$v timeout 900 python bench.py --mode syscalls --cell-ms 60 > gpurun_out/sys90_$v.json 2> gpurun_out/sys90_$v.err
done
