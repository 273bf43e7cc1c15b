#!/bin/bash
timeout 900 python bench.py --mode syscalls > gpurun_out/syscalls12.json 2> gpurun_out/syscalls12.err
timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:wc_kernel -c 1 --csv --log-file gpurun_out/ncu12a.csv python tools/prof_wc.py > gpurun_out/ncu12a.log 2>&1; echo rc=$? >> gpurun_out/ncu12a.log
timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none --replay-mode application -k regex:wc_kernel -c 1 --csv --log-file gpurun_out/ncu12b.csv python tools/prof_wc.py > gpurun_out/ncu12b.log 2>&1; echo rc=$? >> gpurun_out/ncu12b.log
