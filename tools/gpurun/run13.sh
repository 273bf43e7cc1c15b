#!/bin/bash
python -c "import inputs; inputs.make_corpus(512, 16<<20)" 2>&1 | tail -1
timeout 120 ncu --metrics gpu__time_duration.sum --clock-control none --cache-control none -k regex:wc_kernel -c 1 python tools/prof_wc.py host 1 > gpurun_out/ncu13a.log 2>&1; echo rc=$? >> gpurun_out/ncu13a.log
timeout 120 ncu --metrics gpu__time_duration.sum --clock-control none --cache-control none -k regex:wc_kernel -c 1 python tools/prof_wc.py device 1 > gpurun_out/ncu13b.log 2>&1; echo rc=$? >> gpurun_out/ncu13b.log
timeout 900 python bench.py --mode syscalls > gpurun_out/syscalls13.json 2> gpurun_out/syscalls13.err
