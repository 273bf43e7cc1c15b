#!/bin/bash
# final round-1 measurements with the final build
timeout 900 python bench.py > gpurun_out/final_bench.json 2> gpurun_out/final_bench.err; echo rc=$? >> gpurun_out/final_bench.err
timeout 900 python bench.py --mode syscalls > gpurun_out/final_sys.json 2> gpurun_out/final_sys.err; echo rc=$? >> gpurun_out/final_sys.err
timeout 900 python bench.py --mode memcached > gpurun_out/final_mc.json 2> gpurun_out/final_mc.err; echo rc=$? >> gpurun_out/final_mc.err
timeout 600 python bench.py --mode mm > gpurun_out/final_mm.json 2> gpurun_out/final_mm.err; echo rc=$? >> gpurun_out/final_mm.err
timeout 600 python bench.py --mode fig8 > gpurun_out/final_fig8.json 2> gpurun_out/final_fig8.err; echo rc=$? >> gpurun_out/final_fig8.err
timeout 600 python bench.py --mode fig9 > gpurun_out/final_fig9.json 2> gpurun_out/final_fig9.err; echo rc=$? >> gpurun_out/final_fig9.err
