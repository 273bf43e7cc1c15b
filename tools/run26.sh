#!/bin/bash
ZC_THREADS=512 timeout 300 python tools/zc_probe.py > gpurun_out/zc26.jsonl 2> gpurun_out/zc26.err
ZC_THREADS=256 timeout 300 python tools/zc_probe.py >> gpurun_out/zc26.jsonl 2>> gpurun_out/zc26.err
