#!/bin/bash
# token scan: 24 warps (80 registers) vs 28 warps (72 registers) per SM
cd "$GRAFT_REPO_ROOT" || exit 1
O=gpurun_out
L=paper_conf_isca_veselybblor18_b200
for rep in 1 2; do
  SCAN_AB_CELLS="token:768:256,dfa:704:256" timeout 300 python tools/scan_ab.py 20 | sed 's/^{/{"lib": "maxt768", /' >> $O/r02_tok896.jsonl
  GSYS_LIB=$PWD/$L/libgsys_t896.so SCAN_AB_CELLS="token:896:256,token:768:256,token:640:256" timeout 300 python tools/scan_ab.py 20 | sed 's/^{/{"lib": "maxt896", /' >> $O/r02_tok896.jsonl
done
cat $O/r02_tok896.jsonl
