#!/bin/bash
timeout 900 python bench.py --mode syscalls > gpurun_out/sys69.json 2> gpurun_out/sys69.err; echo rc=$? >> gpurun_out/sys69.err
timeout 900 python bench.py > gpurun_out/bench69.json 2> gpurun_out/bench69.err; echo rc=$? >> gpurun_out/bench69.err
timeout 900 python bench.py --mode memcached > gpurun_out/mc69.json 2> gpurun_out/mc69.err; echo rc=$? >> gpurun_out/mc69.err
