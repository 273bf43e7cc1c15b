#!/bin/bash
timeout 1500 python -m pytest tests -m gpu -q -x > gpurun_out/pytest32.log 2>&1; echo rc=$? >> gpurun_out/pytest32.log
timeout 900 python bench.py --mode syscalls > gpurun_out/sys32.json 2> gpurun_out/sys32.err; echo rc=$? >> gpurun_out/sys32.err
