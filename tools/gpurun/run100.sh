#!/bin/bash
timeout 1500 python -m pytest tests -m gpu -q -x > gpurun_out/pytest100.log 2>&1; echo rc=$? >> gpurun_out/pytest100.log
timeout 900 python bench.py --mode memcached > gpurun_out/mc100.json 2> gpurun_out/mc100.err; echo rc=$? >> gpurun_out/mc100.err
