#!/bin/bash
set -x
timeout 900 python -m pytest tests -m gpu -q > gpurun_out/pytest11.log 2>&1; echo rc=$? >> gpurun_out/pytest11.log
timeout 300 python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/smoke11.log 2>&1; echo rc=$? >> gpurun_out/smoke11.log
timeout 600 python bench.py > gpurun_out/bench11.json 2> gpurun_out/bench11.err
timeout 600 python bench.py --impl reference > gpurun_out/bench11_ref.json 2> gpurun_out/bench11_ref.err
ncu --query-metrics 2>/dev/null | grep -iE "pcie|sysmem|nvlrx|nvltx" > gpurun_out/ncu_metrics_pcie.txt
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches11.csv python bench.py --steps 2 --warmup 1 --no-extras --no-cpu-baseline > gpurun_out/ncu_bench11.log 2>&1; echo rc=$? >> gpurun_out/ncu_bench11.log
timeout 900 ncu --set full --clock-control none --import-source on -k regex:scan_kernel -s 1 -c 1 -o gpurun_out/prof_scan11 python tools/prof_scan.py > gpurun_out/ncu_scan11.log 2>&1; echo rc=$? >> gpurun_out/ncu_scan11.log
