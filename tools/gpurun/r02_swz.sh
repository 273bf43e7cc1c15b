#!/bin/bash
# DFA scan with one swizzled tensor copy per tile vs per-lane cp.async staging: scan tests, A/B
cd "$GRAFT_REPO_ROOT" || exit 1
O=gpurun_out
timeout 900 python -m pytest tests -m gpu -x -q -k "scan or dense or degenerate" > $O/r02_swz_tests.log 2>&1; tail -2 $O/r02_swz_tests.log
for rep in 1 2; do
  GSYS_SCAN_SWZ=0 SCAN_AB_CELLS="dfa:1024:256" timeout 300 python tools/scan_ab.py 20 | sed 's/^{/{"staging": "lanes", /' >> $O/r02_swz.jsonl
  SCAN_AB_CELLS="dfa:1024:256,dfa:1024:1024" timeout 300 python tools/scan_ab.py 20 | sed 's/^{/{"staging": "tensor_swz", /' >> $O/r02_swz.jsonl
done
cat $O/r02_swz.jsonl
