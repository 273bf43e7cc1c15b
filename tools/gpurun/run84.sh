#!/bin/bash
timeout 1500 python -m pytest tests -m gpu -q -x > gpurun_out/pytest84.log 2>&1; echo rc=$? >> gpurun_out/pytest84.log
timeout 900 python bench.py > gpurun_out/bench84.json 2> gpurun_out/bench84.err; echo rc=$? >> gpurun_out/bench84.err
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --cache-control none --csv --log-file gpurun_out/launches84.csv python bench.py --steps 2 --warmup 1 --no-extras --no-cpu-baseline > gpurun_out/ncu84.log 2>&1; echo rc=$? >> gpurun_out/ncu84.log
timeout 1500 ncu --set full --import-source on --clock-control none --cache-control none --replay-mode application -k regex:wc_kernel -c 1 -o gpurun_out/prof_wc84 python tools/prof_wc.py host 64 > gpurun_out/ncu_wc84.log 2>&1; echo rc=$? >> gpurun_out/ncu_wc84.log
