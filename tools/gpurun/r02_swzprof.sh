#!/bin/bash
# ncu --set full of the swizzled-TMA DFA scan (base-unit raw page too), then the bench line
cd "$GRAFT_REPO_ROOT" || exit 1
O=gpurun_out
timeout 900 ncu --set full --import-source on --clock-control none -k regex:'^.*scan_kernel' -c 1 -o $O/r02_scan_swz -f python tools/prof_scan.py > $O/r02_scan_swz_ncu.out 2>&1; echo "ncu rc=$?"
ncu -i $O/r02_scan_swz.ncu-rep --page raw --csv --print-units base > $O/r02_scan_swz_raw.csv 2>/dev/null
timeout 600 python bench.py > $O/r02l4_bench.json 2> $O/r02l4_bench.err; echo "bench rc=$?"
