#!/bin/bash
timeout 300 python tools/zc_probe.py > gpurun_out/zc8.jsonl 2> gpurun_out/zc8.err
out=gpurun_out/sweep8.jsonl; : > $out
python -c "import inputs; inputs.make_corpus(512, 16<<20)" 2>&1 | tail -1
GSYS_WC_HOSTBUF=0 GSYS_THREADS=12 timeout 120 python tools/sweep.py --staging host --chunk-kib 256 >> $out 2>>gpurun_out/sweep8.err
GSYS_THREADS=12 timeout 120 python tools/sweep.py --staging host --chunk-kib 256 >> $out 2>>gpurun_out/sweep8.err
