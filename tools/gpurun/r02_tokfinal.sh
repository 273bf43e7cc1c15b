#!/bin/bash
# final token scan (32 warps, one staged tile per warp, two lookups per round): full GPU suite,
# A/B against the DFA, ncu --set full capture
cd "$GRAFT_REPO_ROOT" || exit 1
O=gpurun_out
timeout 1200 python -m pytest tests -m gpu -x -q > $O/r02tf_gputest.log 2>&1; tail -2 $O/r02tf_gputest.log
SCAN_AB_CELLS="token:1024:256,dfa:704:256,token:1024:256,dfa:704:256" timeout 300 python tools/scan_ab.py 20 > $O/r02_tok_final_ab.jsonl; cat $O/r02_tok_final_ab.jsonl
timeout 900 ncu --set full --import-source on --clock-control none -k regex:scan_tok_kernel -c 1 -o $O/r02_scan_tokf -f python tools/prof_scan.py token > $O/r02_scan_tokf_ncu.out 2>&1; echo "ncu rc=$?"
