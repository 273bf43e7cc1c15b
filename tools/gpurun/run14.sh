#!/bin/bash
timeout 900 python -m pytest tests -m gpu -q > gpurun_out/pytest14.log 2>&1; echo rc=$? >> gpurun_out/pytest14.log
timeout 900 python bench.py --mode syscalls > gpurun_out/syscalls14.json 2> gpurun_out/syscalls14.err
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --cache-control none --csv --log-file gpurun_out/launches14.csv python bench.py --steps 2 --warmup 1 --no-extras --no-cpu-baseline > gpurun_out/ncu14.log 2>&1; echo rc=$? >> gpurun_out/ncu14.log
