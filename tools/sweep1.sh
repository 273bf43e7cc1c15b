#!/bin/bash
# first performance sweep on the B200 box
out=gpurun_out/sweep1.jsonl
: > $out
python -c "import inputs; inputs.make_corpus(512, 16<<20)" 2>&1 | tail -1
for t in 4 8 12 14; do
  GSYS_THREADS=$t timeout 120 python tools/sweep.py >> $out 2>>gpurun_out/sweep1.err
done
for c in 64 1024 4096; do
  GSYS_THREADS=12 timeout 120 python tools/sweep.py --chunk-kib $c >> $out 2>>gpurun_out/sweep1.err
done
GSYS_THREADS=12 timeout 120 python tools/sweep.py --blocks 148 >> $out 2>>gpurun_out/sweep1.err
GSYS_THREADS=12 timeout 120 python tools/sweep.py --blocks 1184 >> $out 2>>gpurun_out/sweep1.err
GSYS_THREADS=12 timeout 120 python tools/sweep.py --merge 0 >> $out 2>>gpurun_out/sweep1.err
GSYS_THREADS=12 timeout 120 python tools/sweep.py --cmax 1 >> $out 2>>gpurun_out/sweep1.err
timeout 600 python bench.py > gpurun_out/bench1.json 2> gpurun_out/bench1.err
cat $out
