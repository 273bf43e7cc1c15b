#!/bin/bash
# HBM DFA scan: 24 warps double-buffered (default) vs up to 32 warps with one staged tile per warp
# (the 129-column table then fits beside the staging)
cd "$GRAFT_REPO_ROOT" || exit 1
O=gpurun_out
L=paper_conf_isca_veselybblor18_b200
for rep in 1 2; do
  SCAN_AB_CELLS="dfa:768:256" timeout 300 python tools/scan_ab.py 20 | sed 's/^{/{"lib": "maxt768_nbuf2", /' >> $O/r02_dfa32.jsonl
  GSYS_LIB=$PWD/$L/libgsys_d1024.so SCAN_AB_CELLS="dfa:1024:256,dfa:896:256,dfa:768:256" timeout 300 python tools/scan_ab.py 20 | sed 's/^{/{"lib": "maxt1024_nbuf1", /' >> $O/r02_dfa32.jsonl
  GSYS_LIB=$PWD/$L/libgsys_d1024b2.so SCAN_AB_CELLS="dfa:1024:256,dfa:896:256" timeout 300 python tools/scan_ab.py 20 | sed 's/^{/{"lib": "maxt1024_nbuf2", /' >> $O/r02_dfa32.jsonl
done
cat $O/r02_dfa32.jsonl
