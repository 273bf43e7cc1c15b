#!/bin/bash
timeout 900 python bench.py --mode syscalls > gpurun_out/sys30.json 2> gpurun_out/sys30.err; echo rc=$? >> gpurun_out/sys30.err
