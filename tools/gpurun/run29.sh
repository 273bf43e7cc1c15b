#!/bin/bash
timeout 900 python bench.py --mode memcached > gpurun_out/mc29.json 2> gpurun_out/mc29.err
timeout 900 python bench.py --mode mm > gpurun_out/mm29.json 2> gpurun_out/mm29.err
