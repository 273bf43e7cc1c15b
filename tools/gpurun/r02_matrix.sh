#!/bin/bash
# config-2 syscall matrix with the final library
cd "$GRAFT_REPO_ROOT" || exit 1
O=gpurun_out
timeout 1200 python bench.py --mode syscalls > $O/r02m_syscalls.json 2> $O/r02m_syscalls.err; echo "rc=$?"; tail -c 300 $O/r02m_syscalls.json
