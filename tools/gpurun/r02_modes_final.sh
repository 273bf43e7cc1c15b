#!/bin/bash
# configs 4 and 5, Fig 8 and Fig 9 with the final library
cd "$GRAFT_REPO_ROOT" || exit 1
O=gpurun_out
for m in memcached mm fig8 fig9; do
  timeout 900 python bench.py --mode $m > $O/r02mf_$m.json 2> $O/r02mf_$m.err; echo "$m rc=$?"; tail -c 200 $O/r02mf_$m.json; echo
done
