#!/bin/bash
# token scan: lookups per round (ILP) x warps per SM x staged tiles per warp
cd "$GRAFT_REPO_ROOT" || exit 1
O=gpurun_out
L=paper_conf_isca_veselybblor18_b200
for rep in 1 2; do
  GSYS_LIB=$PWD/$L/libgsys_a.so SCAN_AB_CELLS="token:1024:256" timeout 300 python tools/scan_ab.py 20 | sed 's/^{/{"lib": "maxt1024_nbuf1_ilp2", /' >> $O/r02_tokilp.jsonl
  GSYS_LIB=$PWD/$L/libgsys_b.so SCAN_AB_CELLS="token:1024:256" timeout 300 python tools/scan_ab.py 20 | sed 's/^{/{"lib": "maxt1024_nbuf1_ilp4", /' >> $O/r02_tokilp.jsonl
  GSYS_LIB=$PWD/$L/libgsys_c.so SCAN_AB_CELLS="token:896:256" timeout 300 python tools/scan_ab.py 20 | sed 's/^{/{"lib": "maxt896_nbuf2_ilp4", /' >> $O/r02_tokilp.jsonl
  GSYS_LIB=$PWD/$L/libgsys_d.so SCAN_AB_CELLS="token:896:256" timeout 300 python tools/scan_ab.py 20 | sed 's/^{/{"lib": "maxt896_nbuf1_ilp4", /' >> $O/r02_tokilp.jsonl
  SCAN_AB_CELLS="dfa:704:256" timeout 300 python tools/scan_ab.py 20 | sed 's/^{/{"lib": "default", /' >> $O/r02_tokilp.jsonl
done
cat $O/r02_tokilp.jsonl
