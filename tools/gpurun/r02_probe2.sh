#!/bin/bash
cd "$GRAFT_REPO_ROOT" || exit 1
O=gpurun_out
timeout 300 python -m pytest tests -m gpu -x -q -k "poll_storm" > $O/r02_poll.log 2>&1; tail -2 $O/r02_poll.log
nvcc -O3 -std=c++17 -gencode arch=compute_100a,code=sm_100a -o /tmp/b200_probes tools/probes/b200_probes.cu && timeout 300 /tmp/b200_probes > $O/r02_probes.jsonl 2>&1; tail -6 $O/r02_probes.jsonl
timeout 600 python tools/config1_profile.py > $O/r02_config1_profile.jsonl 2>&1; cat $O/r02_config1_profile.jsonl
