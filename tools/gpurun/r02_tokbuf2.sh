#!/bin/bash
# token scan with two lookups per round: 28 warps double-buffered vs 32 warps single-buffered
cd "$GRAFT_REPO_ROOT" || exit 1
O=gpurun_out
L=paper_conf_isca_veselybblor18_b200
for rep in 1 2; do
  GSYS_LIB=$PWD/$L/libgsys_t896.so SCAN_AB_CELLS="token:896:256" timeout 300 python tools/scan_ab.py 20 | sed 's/^{/{"lib": "x2_maxt896_nbuf2", /' >> $O/r02_tokbuf2.jsonl
  GSYS_LIB=$PWD/$L/libgsys_t1024s.so SCAN_AB_CELLS="token:1024:256" timeout 300 python tools/scan_ab.py 20 | sed 's/^{/{"lib": "x2_maxt1024_nbuf1", /' >> $O/r02_tokbuf2.jsonl
  SCAN_AB_CELLS="token:768:256,dfa:704:256" timeout 300 python tools/scan_ab.py 20 | sed 's/^{/{"lib": "x2_maxt768_nbuf2", /' >> $O/r02_tokbuf2.jsonl
done
cat $O/r02_tokbuf2.jsonl
