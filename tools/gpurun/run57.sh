#!/bin/bash
timeout 900 python -m pytest tests -q -m gpu > gpurun_out/pytest57.log 2>&1; echo rc=$? >> gpurun_out/pytest57.log
timeout 900 python bench.py --mode memcached > gpurun_out/mc57.json 2> gpurun_out/mc57.err
