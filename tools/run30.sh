#!/bin/bash
timeout 600 python -m pytest tests/test_gpu_next.py -m gpu -q -x > gpurun_out/pytest30.log 2>&1; echo rc=$? >> gpurun_out/pytest30.log
timeout 900 python bench.py --mode memcached > gpurun_out/mc30.json 2> gpurun_out/mc30.err
