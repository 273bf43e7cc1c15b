#!/bin/bash
# last verification of the round: full GPU suite, smoke, default bench line
cd "$GRAFT_REPO_ROOT" || exit 1
O=gpurun_out
timeout 1200 python -m pytest tests -m gpu -x -q > $O/r02l_gputest.log 2>&1; tail -2 $O/r02l_gputest.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $O/r02l_smoke.out 2>&1; echo "smoke rc=$?"
timeout 600 python bench.py > $O/r02l_bench.json 2> $O/r02l_bench.err; echo "bench rc=$?"; tail -c 200 $O/r02l_bench.json
