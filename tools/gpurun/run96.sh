#!/bin/bash
for n in 4 8; do
  GSYS_BENCH_ONE_GPU=1 timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node $n --master-addr 127.0.0.1 --master-port 2954$n bench.py --gpus $n --steps 3 --warmup 3 --no-cpu-baseline --no-extras > gpurun_out/n${n}_96.json 2> gpurun_out/n${n}_96.err; echo rc=$? >> gpurun_out/n${n}_96.err
done
