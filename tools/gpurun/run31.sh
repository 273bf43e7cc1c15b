#!/bin/bash
timeout 900 python -m pytest tests -m gpu -q -x -k "getrusage or mm or signal or memcached or inline" > gpurun_out/pytest31.log 2>&1; echo rc=$? >> gpurun_out/pytest31.log
timeout 900 python bench.py --mode syscalls > gpurun_out/sys31.json 2> gpurun_out/sys31.err; echo rc=$? >> gpurun_out/sys31.err
