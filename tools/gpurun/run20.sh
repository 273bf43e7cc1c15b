#!/bin/bash
GSYS_SCAN_LD=0 timeout 300 python tools/zc_probe2.py > gpurun_out/zc20.jsonl 2> gpurun_out/zc20.err
GSYS_SCAN_LD=1 timeout 300 python tools/zc_probe2.py >> gpurun_out/zc20.jsonl 2>> gpurun_out/zc20.err
