#!/bin/bash
# 32-warp single-buffered DFA scan as the default: full GPU suite, A/B, ncu --set full capture
cd "$GRAFT_REPO_ROOT" || exit 1
O=gpurun_out
timeout 1200 python -m pytest tests -m gpu -x -q > $O/r02d_gputest.log 2>&1; tail -2 $O/r02d_gputest.log
SCAN_AB_CELLS="dfa:1024:256,token:1024:256,dfa:1024:256,token:1024:256" timeout 300 python tools/scan_ab.py 20 > $O/r02_dfa32_final_ab.jsonl; cat $O/r02_dfa32_final_ab.jsonl
timeout 900 ncu --set full --import-source on --clock-control none -k regex:'^.*scan_kernel' -c 1 -o $O/r02_scan_dfa32 -f python tools/prof_scan.py > $O/r02_scan_dfa32_ncu.out 2>&1; echo "ncu rc=$?"
