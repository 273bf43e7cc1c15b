#!/bin/bash
python -c "import inputs; inputs.make_corpus(512, 16<<20)" 2>&1 | tail -1
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --cache-control none --csv --log-file gpurun_out/launches15.csv python bench.py --steps 2 --warmup 1 --no-extras --no-cpu-baseline > gpurun_out/ncu15.log 2>&1; echo rc=$? >> gpurun_out/ncu15.log
timeout 600 python bench.py > gpurun_out/bench15.json 2> gpurun_out/bench15.err
