#!/bin/bash
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke77.log 2>&1; echo rc=$? >> gpurun_out/smoke77.log
GSYS_BENCH_ONE_GPU=1 timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29533 bench.py --gpus 2 --steps 3 --warmup 3 --no-cpu-baseline > gpurun_out/n2_77.json 2> gpurun_out/n2_77.err; echo rc=$? >> gpurun_out/n2_77.err
timeout 600 python bench.py --impl reference --steps 2 --warmup 1 > gpurun_out/ref77.json 2> gpurun_out/ref77.err; echo rc=$? >> gpurun_out/ref77.err
