#!/bin/bash
cd "$GRAFT_REPO_ROOT" || exit 1
O=gpurun_out
timeout 1200 python -m pytest tests -m gpu -x -q > $O/r02_gputest_split.log 2>&1; tail -3 $O/r02_gputest_split.log
for sp in 0 128; do GSYS_SPLIT_KB=$sp timeout 300 python tools/config1_sweep.py > $O/r02_config1_split$sp.jsonl 2>&1; echo "split=$sp"; cat $O/r02_config1_split$sp.jsonl; done
for c in 256 64; do timeout 120 python tools/config1_timeline.py $c host; done
timeout 600 python bench.py --no-cpu-baseline > $O/r02_bench_split.json 2> $O/r02_bench_split.err; python -c "
import json; d=json.loads(open('$O/r02_bench_split.json').read().strip().splitlines()[-1]); print(d['value'], d['roofline']['frac'], d['secondary']['config1_16MiB'], d['service_path'])"
