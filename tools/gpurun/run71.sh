#!/bin/bash
# A/B on one box: acquire polls (default) vs relaxed polls + fence, wordcount host staging
python -c "import inputs; inputs.make_corpus(512, 16<<20)" > /dev/null 2>&1
for i in 1 2 3; do
  timeout 120 python tools/sweep.py --staging host --chunk-kib 256 --blocks 296 --steps 5 | sed "s/^{/{\"v\":\"acquire\",/" >> gpurun_out/ab71.jsonl
  GSYS_LIB=$PWD/tools/variants/libgsys_relaxedpoll.so timeout 120 python tools/sweep.py --staging host --chunk-kib 256 --blocks 296 --steps 5 | sed 's/^{/{"v":"relaxed",/' >> gpurun_out/ab71.jsonl
done
