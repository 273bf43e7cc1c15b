#!/bin/bash
# N > 1 path of bench.py on a one-GPU box: 2 and 4 ranks on cuda:0 over gloo (GSYS_BENCH_ONE_GPU=1)
python -c "import inputs; inputs.make_corpus(512, 16<<20)" > /dev/null 2>&1
GSYS_BENCH_ONE_GPU=1 timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29517 bench.py --gpus 2 --steps 3 --warmup 3 > gpurun_out/bench48_n2.json 2> gpurun_out/bench48_n2.err; echo rc=$? >> gpurun_out/bench48_n2.err
GSYS_BENCH_ONE_GPU=1 timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 4 --master-addr 127.0.0.1 --master-port 29518 bench.py --gpus 4 --steps 3 --warmup 3 --no-cpu-baseline > gpurun_out/bench48_n4.json 2> gpurun_out/bench48_n4.err; echo rc=$? >> gpurun_out/bench48_n4.err
timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29519 bench.py --impl reference --gpus 2 --steps 2 --warmup 1 > gpurun_out/bench48_ref2.json 2> gpurun_out/bench48_ref2.err; echo rc=$? >> gpurun_out/bench48_ref2.err
