#!/bin/bash
python -c "import inputs; inputs.make_corpus(512, 16<<20)" > /dev/null 2>&1
timeout 900 python -m pytest tests -q -m gpu > gpurun_out/pytest55.log 2>&1; echo rc=$? >> gpurun_out/pytest55.log
for p in 256 4096; do GSYS_POLL_NS_HOST=$p timeout 120 python tools/lat_probe.py >> gpurun_out/lat55.jsonl 2>> gpurun_out/lat55.err; done
timeout 900 python bench.py --mode syscalls > gpurun_out/syscalls55.json 2> gpurun_out/syscalls55.err
timeout 600 python bench.py --no-extras --no-cpu-baseline > gpurun_out/bench55.json 2> gpurun_out/bench55.err
