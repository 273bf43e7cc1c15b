#!/bin/bash
out=gpurun_out/sweep7.jsonl; : > $out
python -c "import inputs; inputs.make_corpus(512, 16<<20)" 2>&1 | tail -1
for c in 256 1024; do
  GSYS_THREADS=12 timeout 120 python tools/sweep.py --staging host --chunk-kib $c >> $out 2>>gpurun_out/sweep7.err
done
GSYS_THREADS=14 timeout 120 python tools/sweep.py --staging host --chunk-kib 256 >> $out 2>>gpurun_out/sweep7.err
GSYS_THREADS=14 timeout 120 python tools/sweep.py --staging host --chunk-kib 512 >> $out 2>>gpurun_out/sweep7.err
timeout 900 python -m pytest tests -m gpu -q -x -k "staging or host or config1 or ragged" > gpurun_out/pytest7.log 2>&1; echo rc=$? >> gpurun_out/pytest7.log
