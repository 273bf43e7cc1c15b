#!/bin/bash
# re-entry sanity: full GPU parity suite + default bench line
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > gpurun_out/smi40.txt 2>&1
timeout 1500 python -m pytest tests -q -m gpu -x > gpurun_out/pytest40.log 2>&1; echo rc=$? >> gpurun_out/pytest40.log
timeout 900 python bench.py > gpurun_out/bench40.json 2> gpurun_out/bench40.err
