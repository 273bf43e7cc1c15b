#!/bin/bash
# ThreadSanitizer over the host service: TSAN-instrumented libgsys preloaded into python
mkdir -p gpurun_out/tsan
LD_PRELOAD=/usr/lib/gcc/x86_64-linux-gnu/13/libtsan.so GSYS_LIB=$PWD/tools/variants/libgsys_tsan.so \
TSAN_OPTIONS="halt_on_error=0 report_signal_unsafe=0 log_path=$PWD/gpurun_out/tsan/tsan history_size=4" \
timeout 1200 python -m pytest tests/test_gpu.py tests/test_gpu_next.py -m gpu -q -x -p no:cacheprovider \
  -k "config1 or matrix or getrusage or coalesc or trace or ebadf or memcached or injected or pull_sizes" \
  > gpurun_out/tsan/pytest.log 2>&1; echo rc=$? >> gpurun_out/tsan/pytest.log
ls -la gpurun_out/tsan >> gpurun_out/tsan/pytest.log
