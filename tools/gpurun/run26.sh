#!/bin/bash
# round-1 re-entry check: parity suite + default bench on a fresh box
timeout 1200 python -m pytest tests -m gpu -q -x > gpurun_out/pytest26.log 2>&1; echo rc=$? >> gpurun_out/pytest26.log
timeout 900 python bench.py > gpurun_out/bench26.json 2> gpurun_out/bench26.err; echo rc=$? >> gpurun_out/bench26.err
