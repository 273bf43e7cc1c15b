#!/bin/bash
python -c "import inputs; inputs.make_corpus(512, 16<<20)" 2>&1 | tail -1
timeout 600 python bench.py > gpurun_out/bench24.json 2> gpurun_out/bench24.err
timeout 600 python bench.py --impl reference > gpurun_out/bench24_ref.json 2> gpurun_out/bench24_ref.err
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --cache-control none --csv --log-file gpurun_out/launches24.csv python bench.py --steps 2 --warmup 1 --no-extras --no-cpu-baseline > gpurun_out/ncu24.log 2>&1; echo rc=$? >> gpurun_out/ncu24.log
timeout 1500 ncu --set full --import-source on --clock-control none --cache-control none --replay-mode application -k regex:wc_kernel -c 1 -o gpurun_out/prof_wc24 python tools/prof_wc.py host 64 > gpurun_out/ncu_wc24.log 2>&1; echo rc=$? >> gpurun_out/ncu_wc24.log
timeout 900 ncu --set full --clock-control none --import-source on -k regex:scan_kernel -s 1 -c 1 -o gpurun_out/prof_scan24 python tools/prof_scan.py > gpurun_out/ncu_scan24.log 2>&1; echo rc=$? >> gpurun_out/ncu_scan24.log
timeout 900 python bench.py --mode syscalls > gpurun_out/syscalls24.json 2> gpurun_out/syscalls24.err
