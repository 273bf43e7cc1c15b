#!/bin/bash
python -c "import inputs; inputs.make_corpus(512, 16<<20)" > /dev/null 2>&1
cat /sys/bus/pci/devices/*/local_cpulist 2>/dev/null | sort | uniq -c > gpurun_out/cpulist49.txt; nproc >> gpurun_out/cpulist49.txt
timeout 600 python -m pytest tests -q -m gpu -x -k "wordcount_config1 or errors or sigsink or signal" > gpurun_out/pytest49.log 2>&1; echo rc=$? >> gpurun_out/pytest49.log
GSYS_BENCH_ONE_GPU=1 timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29517 bench.py --gpus 2 --steps 3 --warmup 3 --no-extras --no-cpu-baseline > gpurun_out/bench49_n2.json 2> gpurun_out/bench49_n2.err; echo rc=$? >> gpurun_out/bench49_n2.err
timeout 600 python bench.py --no-extras --no-cpu-baseline > gpurun_out/bench49_n1.json 2> gpurun_out/bench49_n1.err
