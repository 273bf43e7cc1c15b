#!/bin/bash
python -c "import inputs; inputs.make_corpus(512, 16<<20)" > /dev/null 2>&1
for v in 0 1; do
  GSYS_BIG_ALONE=$v timeout 300 python tools/config1_profile.py | head -1 | sed "s/^{/{\"big_alone\":$v,/" >> gpurun_out/big94.jsonl 2>&1
  for st in host device; do
    GSYS_BIG_ALONE=$v timeout 120 python tools/sweep.py --staging $st --chunk-kib 256 --blocks 148 --steps 5 | sed "s/^{/{\"big_alone\":$v,/" >> gpurun_out/big94.jsonl 2>&1
  done
done
