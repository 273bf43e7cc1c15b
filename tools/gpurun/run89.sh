#!/bin/bash
timeout 1500 python -m pytest tests -m gpu -q -x > gpurun_out/pytest89.log 2>&1; echo rc=$? >> gpurun_out/pytest89.log
timeout 900 python bench.py --mode syscalls > gpurun_out/sys89.json 2> gpurun_out/sys89.err
