#!/bin/bash
# sleep-hint experiment: learned hint vs none, poll interval 256 vs 1024 ns
timeout 900 python bench.py --mode syscalls --cell-ms 60 > gpurun_out/sys35a.json 2> gpurun_out/sys35a.err
GSYS_SLEEP_HINT=0 timeout 900 python bench.py --mode syscalls --cell-ms 60 > gpurun_out/sys35b.json 2> gpurun_out/sys35b.err
GSYS_SLEEP_HINT=0 GSYS_POLL_NS_HOST=1024 timeout 900 python bench.py --mode syscalls --cell-ms 60 > gpurun_out/sys35c.json 2> gpurun_out/sys35c.err
GSYS_SLEEP_HINT=0 GSYS_POLL_NS_HOST=4096 timeout 900 python bench.py --mode syscalls --cell-ms 60 > gpurun_out/sys35d.json 2> gpurun_out/sys35d.err
