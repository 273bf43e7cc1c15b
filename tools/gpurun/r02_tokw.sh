#!/bin/bash
# warp-cooperative token scan (tokw) vs the byte DFA on 1 GiB of HBM text, then the GPU scan tests
cd "$GRAFT_REPO_ROOT" || exit 1
O=gpurun_out
SCAN_AB_CELLS="token:640:256,token:768:256,dfa:704:256,token:768:256,dfa:704:256" timeout 600 python tools/scan_ab.py 20 > $O/r02_tokw_ab.jsonl 2> $O/r02_tokw_ab.err
cat $O/r02_tokw_ab.jsonl; tail -3 $O/r02_tokw_ab.err
timeout 900 ncu --set full --import-source on --clock-control none -k regex:scan_tok_kernel -c 1 -o $O/r02_scan_tokw -f python tools/prof_scan.py token > $O/r02_scan_tokw_ncu.out 2>&1; echo "ncu rc=$?"
timeout 900 python -m pytest tests -m gpu -x -q -k "scan or wordcount or fuzz or degenerate or token" > $O/r02_tokw_tests.log 2>&1; tail -3 $O/r02_tokw_tests.log
