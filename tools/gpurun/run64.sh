#!/bin/bash
timeout 900 python bench.py > gpurun_out/bench64.json 2> gpurun_out/bench64.err; echo rc=$? >> gpurun_out/bench64.err
timeout 900 python bench.py --mode memcached > gpurun_out/mc64.json 2> gpurun_out/mc64.err; echo rc=$? >> gpurun_out/mc64.err
