#!/bin/bash
timeout 1200 python -m pytest tests -m gpu -q -x -k "wordcount or census" > gpurun_out/pytest28.log 2>&1; echo rc=$? >> gpurun_out/pytest28.log
T=14 timeout 200 python tools/contend_probe.py > gpurun_out/contend28.jsonl 2> gpurun_out/contend28.err
T=6 timeout 200 python tools/contend_probe.py >> gpurun_out/contend28.jsonl 2>> gpurun_out/contend28.err
