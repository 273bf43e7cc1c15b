#!/bin/bash
python -c "import inputs; inputs.make_corpus(512, 16<<20)" > /dev/null 2>&1
for i in 1 2 3; do
  for v in 1 0; do
    GSYS_SHARE_BURSTS=$v timeout 120 python tools/sweep.py --staging host --chunk-kib 256 --blocks 148 --steps 5 | sed "s/^{/{\"share\":$v,/" >> gpurun_out/share91.jsonl 2>&1
  done
done
timeout 1500 python -m pytest tests -m gpu -q -x > gpurun_out/pytest91.log 2>&1; echo rc=$? >> gpurun_out/pytest91.log
