#!/bin/bash
# end-of-round artifacts with the final code: GPU suite, smoke (plain and under ncu), bench line, launch list
cd "$GRAFT_REPO_ROOT" || exit 1
O=gpurun_out
timeout 1200 python -m pytest tests -m gpu -x -q > $O/r02e_gputest.log 2>&1; tail -2 $O/r02e_gputest.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $O/r02e_smoke.out 2>&1; echo "smoke rc=$?"
timeout 600 python bench.py > $O/r02e_bench.json 2> $O/r02e_bench.err; echo "bench rc=$?"
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file $O/r02e_bench_launches.csv python bench.py --steps 2 --warmup 3 --no-extras --no-cpu-baseline > $O/r02e_bench_ncu.out 2>&1; echo "launches rc=$?"
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $O/r02e_smoke_launches.csv python -c "import __graft_entry__ as g; g.smoke()" > $O/r02e_smoke_ncu.out 2>&1; echo "smoke-under-ncu rc=$?"
