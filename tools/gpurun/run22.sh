#!/bin/bash
python -c "import inputs; inputs.make_corpus(512, 16<<20)" 2>&1 | tail -1
timeout 1500 ncu --set full --import-source on --clock-control none --cache-control none --replay-mode application -k regex:wc_kernel -c 1 -o gpurun_out/prof_wc22 python tools/prof_wc.py host 64 > gpurun_out/ncu_wc22.log 2>&1; echo rc=$? >> gpurun_out/ncu_wc22.log
