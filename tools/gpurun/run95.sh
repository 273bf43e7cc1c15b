#!/bin/bash
timeout 1500 python -m pytest tests -m gpu -q -x > gpurun_out/pytest95.log 2>&1; echo rc=$? >> gpurun_out/pytest95.log
timeout 900 python bench.py > gpurun_out/bench95.json 2> gpurun_out/bench95.err; echo rc=$? >> gpurun_out/bench95.err
timeout 900 python bench.py --mode syscalls --cell-ms 60 > gpurun_out/sys95.json 2> gpurun_out/sys95.err
