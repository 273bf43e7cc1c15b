#!/bin/bash
# token scan with the key registers not initialised for empty slots vs the previous build; scan tests
cd "$GRAFT_REPO_ROOT" || exit 1
O=gpurun_out
L=paper_conf_isca_veselybblor18_b200
for rep in 1 2; do
  GSYS_LIB=$PWD/$L/libgsys_base.so SCAN_AB_CELLS="token:1024:256" timeout 300 python tools/scan_ab.py 20 | sed 's/^{/{"lib": "base", /' >> $O/r02_toki.jsonl
  SCAN_AB_CELLS="token:1024:256,dfa:704:256" timeout 300 python tools/scan_ab.py 20 | sed 's/^{/{"lib": "no_key_init", /' >> $O/r02_toki.jsonl
done
cat $O/r02_toki.jsonl
timeout 900 python -m pytest tests -m gpu -x -q -k "scan or wordcount or dense or token or fuzz or degenerate" > $O/r02_toki_tests.log 2>&1; tail -2 $O/r02_toki_tests.log
