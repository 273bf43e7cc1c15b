#!/bin/bash
timeout 1500 python -m pytest tests -m gpu -q -x > gpurun_out/pytest80.log 2>&1; echo rc=$? >> gpurun_out/pytest80.log
timeout 600 python tools/phase_probe.py > gpurun_out/phase80.jsonl 2> gpurun_out/phase80.err
