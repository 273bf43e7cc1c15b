#!/bin/bash
# warp-cooperative work-item pulls + block-copied kernel-scope pulls: GPU tests, syscall matrix
cd "$GRAFT_REPO_ROOT" || exit 1
O=gpurun_out
timeout 1500 python -m pytest tests -m gpu -q -x > $O/r02w_gputest.log 2>&1; tail -3 $O/r02w_gputest.log
timeout 600 python bench.py --mode syscalls > $O/r02w_syscalls.json 2> $O/r02w_syscalls.err; echo "syscalls rc=$?"; tail -c 200 $O/r02w_syscalls.json
timeout 200 python tools/nb_probe.py > $O/r02w_nbprobe.log 2>&1; tail -6 $O/r02w_nbprobe.log
