#!/bin/bash
python -c "import inputs; inputs.make_corpus(512, 16<<20)" > /dev/null 2>&1
for p in 4096 256 512 128 4096; do GSYS_POLL_NS_HOST=$p timeout 300 python bench.py --no-extras --no-cpu-baseline > gpurun_out/bench54_$p.json 2>> gpurun_out/bench54.err; python -c "import json,sys; d=json.load(open('gpurun_out/bench54_$p.json')); print($p, d['value'], d['e2e']['value'], d['parity'])" >> gpurun_out/bench54.txt; done
GSYS_POLL_NS_HOST=512 timeout 120 python tools/lat_probe.py >> gpurun_out/lat54.jsonl 2>> gpurun_out/lat54.err
