#!/bin/bash
# round-2 verification: GPU tests, bench line, ncu launch list of the bench + smoke, one full capture of wc_kernel
cd "$GRAFT_REPO_ROOT" || exit 1
O=gpurun_out
timeout 1200 python -m pytest tests -m gpu -x -q > $O/r02_gputest.log 2>&1; tail -3 $O/r02_gputest.log
timeout 600 python bench.py > $O/r02_bench.json 2> $O/r02_bench.err; tail -c 400 $O/r02_bench.json
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file $O/r02_bench_launches.csv python bench.py --steps 2 --warmup 3 --no-extras --no-cpu-baseline > $O/r02_bench_ncu.out 2>&1; echo "launches rc=$?"
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $O/r02_smoke_launches.csv python -c "import __graft_entry__ as g; g.smoke()" > $O/r02_smoke_ncu.out 2>&1; echo "smoke-under-ncu rc=$?"; tail -2 $O/r02_smoke_ncu.out
timeout 900 ncu --set full --clock-control none --import-source on -k wc_kernel -c 1 -o $O/r02_wc_device -f python tools/prof_wc.py device 64 > $O/r02_wc_ncu.out 2>&1; echo "wc full rc=$?"
