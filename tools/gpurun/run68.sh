#!/bin/bash
timeout 600 python tools/phase_probe.py > gpurun_out/phase68.jsonl 2> gpurun_out/phase68.err
timeout 1500 python -m pytest tests -m gpu -q -x > gpurun_out/pytest68.log 2>&1; echo rc=$? >> gpurun_out/pytest68.log
