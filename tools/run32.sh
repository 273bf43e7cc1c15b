#!/bin/bash
timeout 900 python bench.py --mode fig8 > gpurun_out/fig8.json 2> gpurun_out/fig8.err
timeout 600 python bench.py --mode fig9 > gpurun_out/fig9.json 2> gpurun_out/fig9.err
timeout 900 python bench.py --mode mm > gpurun_out/mm32.json 2> gpurun_out/mm32.err
