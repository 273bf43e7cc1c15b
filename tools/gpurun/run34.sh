#!/bin/bash
timeout 1500 python -m pytest tests -m gpu -q -x > gpurun_out/pytest34.log 2>&1; echo rc=$? >> gpurun_out/pytest34.log
timeout 900 python bench.py --mode syscalls > gpurun_out/sys34.json 2> gpurun_out/sys34.err; echo rc=$? >> gpurun_out/sys34.err
timeout 900 python bench.py > gpurun_out/bench34.json 2> gpurun_out/bench34.err; echo rc=$? >> gpurun_out/bench34.err
