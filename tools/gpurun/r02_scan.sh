#!/bin/bash
cd "$GRAFT_REPO_ROOT" || exit 1
O=gpurun_out
timeout 900 python -m pytest tests -m gpu -x -q -k "scan or wordcount or smoke" > $O/r02_scan_tests.log 2>&1; tail -3 $O/r02_scan_tests.log
timeout 300 python tools/scan_ab.py 10 > $O/r02_scan_ab.jsonl 2>&1; cat $O/r02_scan_ab.jsonl
nvcc -O3 -std=c++17 -gencode arch=compute_100a,code=sm_100a -o /tmp/b200_probes tools/probes/b200_probes.cu && timeout 300 /tmp/b200_probes > $O/r02_probes.jsonl 2>&1; cat $O/r02_probes.jsonl
timeout 300 python tools/config1_sweep.py > $O/r02_config1_sweep.jsonl 2>&1; cat $O/r02_config1_sweep.jsonl
