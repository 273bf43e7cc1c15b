#!/bin/bash
timeout 900 python -m pytest tests -m gpu -q -x > gpurun_out/pytest25.log 2>&1; echo rc=$? >> gpurun_out/pytest25.log
timeout 300 python tools/zc_probe.py > gpurun_out/zc25.jsonl 2> gpurun_out/zc25.err
python -c "import inputs; inputs.make_corpus(512, 16<<20)" 2>&1 | tail -1
timeout 120 python tools/sweep.py --staging host --chunk-kib 256 --blocks 296 > gpurun_out/sweep25.jsonl 2>>gpurun_out/sweep25.err
