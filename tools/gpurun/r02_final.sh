#!/bin/bash
# final-code measurement: default bench line, reference arm, launch lists of the bench and smoke
cd "$GRAFT_REPO_ROOT" || exit 1
O=gpurun_out
timeout 600 python bench.py > $O/r02f_bench.json 2> $O/r02f_bench.err; tail -c 300 $O/r02f_bench.json
timeout 600 python bench.py --impl reference --steps 2 --warmup 1 > $O/r02f_ref.json 2> $O/r02f_ref.err; tail -c 300 $O/r02f_ref.json
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file $O/r02f_bench_launches.csv python bench.py --steps 2 --warmup 3 --no-extras --no-cpu-baseline > $O/r02f_bench_ncu.out 2>&1; echo "launches rc=$?"
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $O/r02f_smoke_launches.csv python -c "import __graft_entry__ as g; g.smoke()" > $O/r02f_smoke_ncu.out 2>&1; echo "smoke-under-ncu rc=$?"
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $O/r02f_smoke.out 2>&1; echo "smoke rc=$?"
