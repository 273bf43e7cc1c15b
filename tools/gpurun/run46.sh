#!/bin/bash
timeout 900 python -m pytest tests -q -m gpu -x -k "wordcount or full_size or errors or trace" > gpurun_out/pytest46.log 2>&1; echo rc=$? >> gpurun_out/pytest46.log
timeout 900 python bench.py > gpurun_out/bench46.json 2> gpurun_out/bench46.err
timeout 900 python bench.py --no-extras --no-cpu-baseline --steps 8 > gpurun_out/bench46b.json 2>> gpurun_out/bench46.err
