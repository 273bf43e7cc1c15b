#!/bin/bash
# token scan: warps per SM x staged tiles per warp (double-buffered 28 warps vs single-buffered 28 / 32)
cd "$GRAFT_REPO_ROOT" || exit 1
O=gpurun_out
L=paper_conf_isca_veselybblor18_b200
for rep in 1 2; do
  GSYS_LIB=$PWD/$L/libgsys_t896.so SCAN_AB_CELLS="token:896:256" timeout 300 python tools/scan_ab.py 20 | sed 's/^{/{"lib": "maxt896_nbuf2", /' >> $O/r02_tokbuf.jsonl
  GSYS_LIB=$PWD/$L/libgsys_t896s.so SCAN_AB_CELLS="token:896:256" timeout 300 python tools/scan_ab.py 20 | sed 's/^{/{"lib": "maxt896_nbuf1", /' >> $O/r02_tokbuf.jsonl
  GSYS_LIB=$PWD/$L/libgsys_t1024s.so SCAN_AB_CELLS="token:1024:256,token:960:256" timeout 300 python tools/scan_ab.py 20 | sed 's/^{/{"lib": "maxt1024_nbuf1", /' >> $O/r02_tokbuf.jsonl
done
cat $O/r02_tokbuf.jsonl
