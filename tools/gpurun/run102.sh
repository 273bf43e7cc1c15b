#!/bin/bash
# header written by warp 0, sent by warp 1: with per-thread fences before Bar1 the replies must be exact
for i in 1 2 3; do timeout 900 python -m pytest tests/test_gpu_next.py -m gpu -q -x -k memcached > gpurun_out/pytest102_$i.log 2>&1; echo rc=$? >> gpurun_out/pytest102_$i.log; done
timeout 1500 python -m pytest tests -m gpu -q -x > gpurun_out/pytest102.log 2>&1; echo rc=$? >> gpurun_out/pytest102.log
timeout 900 python bench.py --mode memcached > gpurun_out/mc102.json 2> gpurun_out/mc102.err
timeout 600 python bench.py --mode fig8 > gpurun_out/fig8_102.json 2> gpurun_out/fig8_102.err
