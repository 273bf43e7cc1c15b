#!/bin/bash
# round-1 refresh after the scan rewrite: parity, bench line, launch list, ncu captures, sanitizers
timeout 900 python -m pytest tests -q -m gpu > gpurun_out/pytest45.log 2>&1; echo rc=$? >> gpurun_out/pytest45.log
timeout 900 python bench.py > gpurun_out/bench45.json 2> gpurun_out/bench45.err
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --cache-control none --csv --log-file gpurun_out/launches45.csv python bench.py --steps 2 --warmup 1 --no-extras --no-cpu-baseline > gpurun_out/ncu45.log 2>&1; echo rc=$? >> gpurun_out/ncu45.log
timeout 600 ncu --set full --clock-control none --import-source on -k regex:scan_kernel -s 1 -c 1 -o gpurun_out/prof_scan45 python tools/scan_bench.py 512 256 2 > gpurun_out/ncu_scan45.log 2>&1; echo rc=$? >> gpurun_out/ncu_scan45.log
timeout 1500 ncu --set full --import-source on --clock-control none --cache-control none --replay-mode application -k regex:wc_kernel -c 1 -o gpurun_out/prof_wc45 python tools/prof_wc.py host 64 > gpurun_out/ncu_wc45.log 2>&1; echo rc=$? >> gpurun_out/ncu_wc45.log
for t in memcheck racecheck synccheck; do timeout 600 compute-sanitizer --tool $t python tools/sanitize_small.py > gpurun_out/san45_$t.log 2>&1; echo rc=$? >> gpurun_out/san45_$t.log; done
