#!/bin/bash
# full GPU suite on the rebased-DFA build + one ncu --set full capture of scan_kernel (1 GiB HBM text)
cd "$GRAFT_REPO_ROOT" || exit 1
O=gpurun_out
timeout 1200 python -m pytest tests -m gpu -x -q > $O/r02s_gputest.log 2>&1; tail -2 $O/r02s_gputest.log
timeout 900 ncu --set full --import-source on --clock-control none -k regex:scan_kernel -c 1 -o $O/r02_scan_dfa2 -f python tools/prof_scan.py > $O/r02_scan_dfa2_ncu.out 2>&1; echo "dfa rc=$?"
