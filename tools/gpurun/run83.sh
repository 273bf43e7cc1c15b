#!/bin/bash
python -c "import inputs; inputs.make_corpus(512, 16<<20)" > /dev/null 2>&1
for i in 1 2 3; do
  for b in 148 296 222; do
    timeout 120 python tools/sweep.py --staging host --chunk-kib 256 --blocks $b --steps 5 >> gpurun_out/blocks83.jsonl 2>&1
  done
done
