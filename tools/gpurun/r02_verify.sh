#!/bin/bash
# round-2 verification: GPU tests, smoke (plain and under ncu), bench line, launch list, prefetch
cd "$GRAFT_REPO_ROOT" || exit 1
O=gpurun_out
timeout 1500 python -m pytest tests -m gpu -q > $O/r02v_gputest.log 2>&1; tail -2 $O/r02v_gputest.log
timeout 300 python -c "import __graft_entry__ as g; g.build(); g.smoke()" > $O/r02v_smoke.log 2>&1; tail -1 $O/r02v_smoke.log
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $O/r02v_smoke_launches.csv python -c "import __graft_entry__ as g; g.smoke()" > $O/r02v_smoke_ncu.out 2>&1; echo "smoke-under-ncu rc=$?"
timeout 600 python bench.py > $O/r02v_bench.json 2> $O/r02v_bench.err; tail -c 300 $O/r02v_bench.json
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file $O/r02v_bench_launches.csv python bench.py --steps 2 --warmup 3 --no-extras --no-cpu-baseline > $O/r02v_bench_ncu.out 2>&1; echo "launches rc=$?"
timeout 300 python bench.py --staging device --no-extras --no-cpu-baseline --steps 3 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read().strip().splitlines()[-1]); print('device-blocking', d['value'])"
