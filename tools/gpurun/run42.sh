#!/bin/bash
# refreshed ncu evidence for the current build: launch list of the bench command, full captures
python -c "import inputs; inputs.make_corpus(512, 16<<20)" > /dev/null 2>&1
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --cache-control none --csv --log-file gpurun_out/launches42.csv python bench.py --steps 2 --warmup 1 --no-extras --no-cpu-baseline > gpurun_out/ncu42.log 2>&1; echo rc=$? >> gpurun_out/ncu42.log
timeout 1500 ncu --set full --import-source on --clock-control none --cache-control none --replay-mode application -k regex:wc_kernel -c 1 -o gpurun_out/prof_wc42 python tools/prof_wc.py host 64 > gpurun_out/ncu_wc42.log 2>&1; echo rc=$? >> gpurun_out/ncu_wc42.log
timeout 900 ncu --set full --clock-control none --import-source on -k regex:scan_kernel -s 1 -c 1 -o gpurun_out/prof_scan42 python tools/prof_scan.py > gpurun_out/ncu_scan42.log 2>&1; echo rc=$? >> gpurun_out/ncu_scan42.log
