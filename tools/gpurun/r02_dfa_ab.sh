#!/bin/bash
# DFA scan A/B on one box: rebased shared-address entries + predicated emission (libgsys.so) vs
# the previous build (libgsys_base.so), alternating, 1 GiB HBM text, 704 threads; then the scan tests
cd "$GRAFT_REPO_ROOT" || exit 1
O=gpurun_out
for rep in 1 2 3; do
  for v in base new; do
    if [ $v = base ]; then L=paper_conf_isca_veselybblor18_b200/libgsys_base.so; else L=paper_conf_isca_veselybblor18_b200/libgsys.so; fi
    GSYS_LIB=$PWD/$L timeout 300 python tools/scan_bench.py 704 256 30 | sed "s/^{/{\"lib\": \"$v\", /" >> $O/r02_dfa_ab.jsonl
  done
done
cat $O/r02_dfa_ab.jsonl
timeout 900 python -m pytest tests -m gpu -x -q -k "scan or wordcount or fuzz or degenerate" > $O/r02_dfa_tests.log 2>&1; tail -3 $O/r02_dfa_tests.log
