#!/bin/bash
# round-2 re-entry check: GPU suite + default bench line + smoke
cd "$GRAFT_REPO_ROOT" || exit 1
O=gpurun_out
timeout 1200 python -m pytest tests -m gpu -x -q > $O/r02c_gputest.log 2>&1; tail -3 $O/r02c_gputest.log
timeout 600 python bench.py > $O/r02c_bench.json 2> $O/r02c_bench.err; tail -c 600 $O/r02c_bench.json
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $O/r02c_smoke.out 2>&1; echo "smoke rc=$?"
