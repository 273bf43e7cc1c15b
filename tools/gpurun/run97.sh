#!/bin/bash
# end-of-session verification of the committed tree
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/smoke97.log 2>&1; echo rc=$? >> gpurun_out/smoke97.log
timeout 1500 python -m pytest tests -m gpu -q -x > gpurun_out/pytest97.log 2>&1; echo rc=$? >> gpurun_out/pytest97.log
timeout 900 python bench.py > gpurun_out/bench97.json 2> gpurun_out/bench97.err; echo rc=$? >> gpurun_out/bench97.err
timeout 600 python bench.py --impl reference > gpurun_out/ref97.json 2> gpurun_out/ref97.err; echo rc=$? >> gpurun_out/ref97.err
