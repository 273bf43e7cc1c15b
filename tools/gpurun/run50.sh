#!/bin/bash
python -c "import inputs; inputs.make_corpus(512, 16<<20)" > /dev/null 2>&1
for i in 1 2; do timeout 600 python bench.py --no-extras --no-cpu-baseline > gpurun_out/bench50_$i.json 2> gpurun_out/bench50_$i.err; done
nvidia-smi -q -d CLOCK,PERFORMANCE > gpurun_out/smi50.txt 2>&1
lscpu > gpurun_out/lscpu50.txt; free -g >> gpurun_out/lscpu50.txt
