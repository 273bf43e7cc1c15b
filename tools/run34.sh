#!/bin/bash
timeout 900 compute-sanitizer --tool racecheck --print-limit 20 python tools/sanitize_small.py > gpurun_out/san_racecheck.log 2>&1; echo rc=$? >> gpurun_out/san_racecheck.log
timeout 900 python -m pytest tests -m gpu -q > gpurun_out/pytest34.log 2>&1; echo rc=$? >> gpurun_out/pytest34.log
