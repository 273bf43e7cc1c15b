#!/bin/bash
cd "$GRAFT_REPO_ROOT" || exit 1
O=gpurun_out
python -c "import inputs; inputs.make_corpus(512, 16 << 20)" > /dev/null 2>&1
timeout 900 ncu --set full --import-source on --clock-control none -k regex:scan_tok_kernel -c 1 -o $O/r02_scan_tokw -f python tools/prof_scan.py token > $O/r02_scan_tokw_ncu.out 2>&1; echo "tok rc=$?"
